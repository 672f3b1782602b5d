"""Profiling driver (not a benchmark): run the A1-A4 chain on a config a few times so ncu can capture one launch
of a chosen kernel, e.g.
  ncu --set full --import-source on -k regex:k_bbv -s 2 -c 1 -o gpurun_out/k1 python profiles/run_chain.py 5"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tracegen as tg  # noqa: E402
from paper_conf_micro_liusc23_b200 import DeviceTrace, Photon  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 5
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
ph = Photon(0)
g = tg.Generator(cfg)
d = DeviceTrace.from_host(g.trace(), ph.device)
ph.analyse(d)  # checked once: learns the table / pair capacities (an unchecked call never retries)
for _ in range(reps):
    ph.analyse(d, check=False)
torch.cuda.synchronize()
