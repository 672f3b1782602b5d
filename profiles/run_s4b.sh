python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "bbv or k1 or group or chain or analyse or debug or smoke or config or random or empty" > gpurun_out/gputest_s4b.log 2>&1; tail -1 gpurun_out/gputest_s4b.log
bash profiles/ab.sh 5 r2 r4 r8
for c in 3 4 2; do for v in base r4; do if [ $v = base ]; then python profiles/time_chain.py $c | sed "s/^/base /"; else PHOTON_LIB_OVERRIDE=$PWD/abvar/libphoton_$v.so python profiles/time_chain.py $c | sed "s/^/$v /"; fi; done; done
