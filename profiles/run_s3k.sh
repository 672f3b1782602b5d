bash profiles/ab.sh 5 xg8 xg32 unr16 xg8u16
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/chain_launches_s3k.csv python profiles/run_chain.py 5 1 > /dev/null 2>&1
python profiles/launch_summary.py gpurun_out/chain_launches_s3k.csv 2>&1
