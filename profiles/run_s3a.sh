python -m pytest tests -m gpu -q -x > gpurun_out/gputest_s3.log 2>&1; tail -3 gpurun_out/gputest_s3.log
python bench.py --skip-cpu > gpurun_out/bench_s3.json 2> gpurun_out/bench_s3.err; tail -2 gpurun_out/bench_s3.err
python profiles/time_k1.py 5 > gpurun_out/timek1_s3.txt 2>&1
