ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed --clock-control none --csv --log-file gpurun_out/chain_launches_s3.csv python profiles/run_chain.py 5 1 > /dev/null 2>&1
python profiles/launch_summary.py gpurun_out/chain_launches_s3.csv 2>&1 | head -60
