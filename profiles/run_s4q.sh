python -m pytest tests -m gpu -q -x --deselect tests/test_sanitizer.py -k "chain or analyse or debug or smoke or errors or out_reuse or config_small or random" > gpurun_out/gputest_s4q.log 2>&1; tail -1 gpurun_out/gputest_s4q.log
for i in 1 2 3; do python profiles/time_chain.py 5; done
