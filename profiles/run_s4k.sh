python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "match or chain or analyse or pool or dist or debug or config or group" > gpurun_out/gputest_s4k.log 2>&1; tail -1 gpurun_out/gputest_s4k.log
for i in 1 2; do python profiles/time_chain.py 5; done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/chain_s4k.csv python profiles/run_chain.py 5 1 > /dev/null 2>&1; python profiles/launch_summary.py gpurun_out/chain_s4k.csv | grep "sort\|total"
