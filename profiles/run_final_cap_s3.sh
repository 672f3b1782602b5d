ncu --profile-from-start off --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/sec_chain.csv python profiles/run_section.py chain > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_s3d.csv python bench.py --steps 2 --warmup 1 --skip-cpu --skip-configs --skip-e2e > gpurun_out/b_under_ncu_s3d.log 2>&1
ls -la gpurun_out/sec_chain.csv gpurun_out/launches_s3d.csv
