python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "stable or debug" > gpurun_out/gputest_s3u.log 2>&1; tail -1 gpurun_out/gputest_s3u.log
python bench.py --skip-cpu --skip-configs --skip-e2e --steps 20 > gpurun_out/b_s3u.json 2>/dev/null
python -c "
import json; d=json.load(open('gpurun_out/b_s3u.json'))
for k in ('a5','a5_c5'): print(k, d[k]['ms_per_step'], d[k]['roofline']['frac'])
"
