python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "bbv or k1 or group or chain or smoke or analyse" > gpurun_out/gputest_s3c.log 2>&1; tail -3 gpurun_out/gputest_s3c.log
python profiles/time_chain.py 5 > gpurun_out/tc_s3c.txt; cat gpurun_out/tc_s3c.txt
