python -m pytest tests -m gpu -q > gpurun_out/gputest_final_s3.log 2>&1; tail -2 gpurun_out/gputest_final_s3.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
bash profiles/run_bench_s3.sh
