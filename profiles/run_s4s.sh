for v in base nv4 nv8; do
  if [ $v = base ]; then ov=""; else ov="PHOTON_LIB_OVERRIDE=$PWD/abvar/libphoton_$v.so"; fi
  env $ov ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/n2_$v.csv python profiles/run_section.py n2 > /dev/null 2>&1
  echo "== $v"; python profiles/launch_summary.py gpurun_out/n2_$v.csv | grep "hash_long\|total"
done
