python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "match or chain or analyse or group or smoke or dist or pool" > gpurun_out/gputest_s3n.log 2>&1; tail -1 gpurun_out/gputest_s3n.log
bash profiles/ab.sh 5 nopdl
