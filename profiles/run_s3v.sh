for v in sthead stpres sthist; do
  PHOTON_LIB_OVERRIDE=$PWD/abvar/libphoton_$v.so ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/a5_$v.csv python profiles/run_section.py a5_c5 > /dev/null 2>&1
  echo "== $v"; python profiles/launch_summary.py gpurun_out/a5_$v.csv | grep "presence\|job_hist\|total"
done
ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/a5_both.csv python profiles/run_section.py a5_c5 > /dev/null 2>&1
echo "== both"; python profiles/launch_summary.py gpurun_out/a5_both.csv | grep "presence\|job_hist\|total"
