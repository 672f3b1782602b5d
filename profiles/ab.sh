#!/bin/bash
# A/B timing probe: alternate the in-tree library with experiment builds in exp/ (same box, same data)
cfg=${1:-5}; shift
for r in 1 2 3; do
  python profiles/time_k1.py $cfg | sed "s/^/base  /"
  for e in "$@"; do PHOTON_LIB_OVERRIDE=$PWD/abvar/libphoton_$e.so python profiles/time_k1.py $cfg | sed "s/^/$e  /"; done
done
