python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "match or chain or analyse or pool or dist" > gpurun_out/gputest_s3l.log 2>&1; tail -1 gpurun_out/gputest_s3l.log
bash profiles/ab.sh 5 xg4 xg8u4 xg4u16
