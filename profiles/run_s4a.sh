python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "bbv or k1 or group or chain or analyse or debug or smoke or config or random or empty" > gpurun_out/gputest_s4a.log 2>&1; tail -1 gpurun_out/gputest_s4a.log
bash profiles/ab.sh 5 st48 st56 u128 nodyn
for c in 3 4 2; do python profiles/time_chain.py $c | sed "s/^/dyn /"; PHOTON_LIB_OVERRIDE=$PWD/abvar/libphoton_nodyn.so python profiles/time_chain.py $c | sed "s/^/nodyn /"; done
