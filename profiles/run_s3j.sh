python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "match or chain or analyse" > gpurun_out/gputest_s3j.log 2>&1; tail -1 gpurun_out/gputest_s3j.log
bash profiles/ab.sh 5 frb1 frb4 noband
