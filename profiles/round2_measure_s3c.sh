# Round-2 session-3 final capture: GPU tests, smoke, per-section DRAM traffic, launch list, K1 ncu.
set -x
python -m pytest tests -m gpu -q > gpurun_out/gputest_s3c_final.log 2>&1; tail -3 gpurun_out/gputest_s3c_final.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_s3c.log 2>&1; tail -2 gpurun_out/smoke_s3c.log
for sec in chain a5 a5_c5 n1 n2 n3; do ncu --profile-from-start off --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/sec_$sec.csv python profiles/run_section.py $sec > /dev/null 2>&1; done
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_s3c.csv python bench.py --steps 2 --warmup 1 --skip-cpu --skip-configs --skip-e2e > gpurun_out/b_under_ncu_s3c.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_bbv3" -c 1 -o gpurun_out/k1_s3c python profiles/run_chain.py 5 1 > /dev/null 2>&1
ls gpurun_out | tail -3
