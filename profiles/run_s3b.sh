python -m pytest tests -m gpu -q --deselect tests/test_sanitizer.py > gpurun_out/gputest_s3b.log 2>&1; tail -3 gpurun_out/gputest_s3b.log
ncu --set full --clock-control none --import-source on -k regex:"k_bbv3" -c 1 -o gpurun_out/k1_s3 python profiles/run_chain.py 5 1 > gpurun_out/k1_s3.log 2>&1; tail -2 gpurun_out/k1_s3.log
