python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "bbv or k1 or group or chain or analyse or debug or smoke or config or random or empty" > gpurun_out/gputest_s3w.log 2>&1; tail -1 gpurun_out/gputest_s3w.log
for c in 3 4 2 5; do
  python profiles/time_chain.py $c | sed "s/^/new /"
  PHOTON_LIB_OVERRIDE=$PWD/abvar/libphoton_k1old.so python profiles/time_chain.py $c | sed "s/^/old /"
done
