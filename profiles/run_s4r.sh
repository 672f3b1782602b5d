python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "match or chain or analyse or pool or dist or debug or config or smoke" > gpurun_out/gputest_s4r.log 2>&1; tail -1 gpurun_out/gputest_s4r.log
for i in 1 2 3; do python profiles/time_chain.py 5; done
