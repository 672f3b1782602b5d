python -m pytest tests/test_debug_build.py -q -x > gpurun_out/gputest_s3o.log 2>&1; tail -15 gpurun_out/gputest_s3o.log
python profiles/time_chain.py 5
