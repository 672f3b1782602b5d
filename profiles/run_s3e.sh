ncu --set full --clock-control none --import-source on -k regex:"k_bbv3" -c 1 -o gpurun_out/k1_v4a python profiles/run_chain.py 5 1 > gpurun_out/k1_v4a.log 2>&1; tail -2 gpurun_out/k1_v4a.log
