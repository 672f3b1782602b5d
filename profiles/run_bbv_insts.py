"""Profiling driver (not a benchmark): photon_bbv_build with warp_insts only (the K1 streaming pass without the
fused de-duplication), a few times."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tracegen as tg  # noqa: E402
from paper_conf_micro_liusc23_b200 import DeviceTrace, Photon  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 5
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
ph = Photon(0)
d = DeviceTrace.from_host(tg.Generator(cfg).trace(), ph.device)
o = {}
for _ in range(reps):
    ph.photon_bbv_build(d, bbv16=False, insts=True, check=False, out=o)
torch.cuda.synchronize()
