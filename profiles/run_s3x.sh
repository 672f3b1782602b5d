for c in 5 3 4; do
  python profiles/time_chain.py $c | sed "s/^/base /"
  for v in a24 a32 a64 a96; do PHOTON_LIB_OVERRIDE=$PWD/abvar/libphoton_$v.so python profiles/time_chain.py $c | sed "s/^/$v /"; done
done
