python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "match or chain or analyse or group or smoke or dist or pool" > gpurun_out/gputest_s3i.log 2>&1; tail -2 gpurun_out/gputest_s3i.log
for i in 1 2; do python profiles/time_chain.py 5; done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/chain_launches_s3i.csv python profiles/run_chain.py 5 1 > /dev/null 2>&1
python profiles/launch_summary.py gpurun_out/chain_launches_s3i.csv 2>&1 | grep -i "band\|filter\|total"
