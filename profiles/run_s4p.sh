python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "match_many or c5_full or chain or analyse" > gpurun_out/gputest_s4p.log 2>&1; tail -1 gpurun_out/gputest_s4p.log
