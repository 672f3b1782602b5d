#!/bin/bash
# A/B timing probe: alternate the in-tree library with experiment builds in abvar/ (same box, same data)
cfg=${1:-5}; shift
probe=${PROBE:-profiles/time_chain.py}
for r in 1 2 3; do
  python $probe $cfg | sed "s/^/base  /"
  for e in "$@"; do PHOTON_LIB_OVERRIDE=$PWD/abvar/libphoton_$e.so python $probe $cfg | sed "s/^/$e  /"; done
done
