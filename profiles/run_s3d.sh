python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "bbv or k1 or group or chain or smoke or analyse" > gpurun_out/gputest_s3d.log 2>&1; tail -2 gpurun_out/gputest_s3d.log
bash profiles/ab.sh 5 v4b v4c nar v4q7 > gpurun_out/ab.txt 2>&1; cat gpurun_out/ab.txt
