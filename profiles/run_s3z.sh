PHOTON_LIB_OVERRIDE=$PWD/abvar/libphoton_tail.so python profiles/run_tail.py 5 2>&1 | tail -3 | sed "s/^/static /"
TAIL_MAP=il PHOTON_LIB_OVERRIDE=$PWD/abvar/libphoton_tailil.so python profiles/run_tail.py 5 2>&1 | tail -3 | sed "s/^/interleaved /"
