python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "bbv or k1 or group or chain or analyse or debug or smoke or config or random or empty" > gpurun_out/gputest_s4e.log 2>&1; tail -1 gpurun_out/gputest_s4e.log
bash profiles/ab.sh 5 nodyn s48 s56 u6
for c in 3 4 2; do python profiles/time_chain.py $c | sed "s/^/base /"; PHOTON_LIB_OVERRIDE=$PWD/abvar/libphoton_nodyn.so python profiles/time_chain.py $c | sed "s/^/nodyn /"; done
