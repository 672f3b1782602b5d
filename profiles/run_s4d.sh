python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "predict or debug" > gpurun_out/gputest_s4d.log 2>&1; tail -1 gpurun_out/gputest_s4d.log
python bench.py --skip-cpu --skip-configs --skip-e2e --steps 20 > gpurun_out/b_s4d.json 2>/dev/null
python -c "
import json; d=json.load(open('gpurun_out/b_s4d.json'))
for k in ('n3','n1','n2'): print(k, d[k]['ms_per_step'], d[k]['roofline']['frac'])
"
ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/sec_n3_s4d.csv python profiles/run_section.py n3 > /dev/null 2>&1; python profiles/launch_summary.py gpurun_out/sec_n3_s4d.csv
