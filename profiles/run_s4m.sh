python -m pytest tests -m gpu -q > gpurun_out/gputest_s4m.log 2>&1; tail -2 gpurun_out/gputest_s4m.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
