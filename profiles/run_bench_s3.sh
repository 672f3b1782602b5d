python bench.py > gpurun_out/bench_s3final.json 2> gpurun_out/bench_s3final.err; tail -3 gpurun_out/bench_s3final.err
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref_s3.json 2> gpurun_out/bench_ref_s3.err; tail -2 gpurun_out/bench_ref_s3.err
