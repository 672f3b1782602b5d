python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "bbv or k1 or group or chain or analyse or debug" > gpurun_out/gputest_s3y.log 2>&1; tail -1 gpurun_out/gputest_s3y.log
bash profiles/ab.sh 5 t256 t512 c1
