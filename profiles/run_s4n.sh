env | grep NCCL
python bench.py --sharded --steps 20 --warmup 3 --skip-cpu --skip-configs --skip-e2e --skip-a5 > gpurun_out/b_sharded.json 2> gpurun_out/b_sharded.err; wc -l gpurun_out/b_sharded.json; head -c 200 gpurun_out/b_sharded.json; echo; tail -3 gpurun_out/b_sharded.err
