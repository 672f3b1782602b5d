for c in 3 4 2; do python profiles/time_chain.py $c | sed "s/^/base /"; PHOTON_LIB_OVERRIDE=$PWD/abvar/libphoton_r2.so python profiles/time_chain.py $c | sed "s/^/r2 /"; done
