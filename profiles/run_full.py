"""Profiling driver (not a benchmark): photon_warp_group_full (N2) on one config, bbv16 precomputed."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tracegen as tg  # noqa: E402
from paper_conf_micro_liusc23_b200 import DeviceTrace, Photon  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 3
ph = Photon(0)
d = DeviceTrace.from_host(tg.Generator(cfg).trace(), ph.device)
b16 = ph.photon_bbv_build(d, bbv16=True, insts=False)["warp_bbv16"]
torch.cuda.synchronize()
o = ph.photon_warp_group_full(d, b16)  # checked: learns the type-table hint
ph.photon_warp_group_full(d, b16, check=False, out=o)  # the steady-state call (small table)
torch.cuda.synchronize()
