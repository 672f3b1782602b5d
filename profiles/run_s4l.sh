python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "bbv or k1 or group or chain or analyse or debug or smoke or config or random or empty" > gpurun_out/gputest_s4l.log 2>&1; tail -1 gpurun_out/gputest_s4l.log
for i in 1 2; do python profiles/time_chain.py 5; done
