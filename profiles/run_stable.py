"""Profiling driver (not a benchmark): run the A5 stability test on one config's timing stream a few times so ncu can
capture its launches, e.g.
  ncu --metrics gpu__time_duration.sum --clock-control none --csv python profiles/run_stable.py 3"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tracegen as tg  # noqa: E402
from paper_conf_micro_liusc23_b200 import DeviceTiming, DeviceTrace, Photon  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 3
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
k1 = int(sys.argv[3]) if len(sys.argv) > 3 else None  # a kernel prefix (C5: 1000 as in bench.py)
ph = Photon(0)
g = tg.Generator(cfg)
k1 = g.n_kernels if k1 is None else k1
d = DeviceTrace.from_host(g.kernels_trace(0, k1), ph.device)
kbb = ph.photon_bbv_build(d, bbv16=False, insts=False, kbb=True)["kernel_bb_insts"]
dt = DeviceTiming.from_host(g.timing(0, k1), ph.device)
o = ph.photon_bb_stable(dt, kbb, 2048)
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(reps):
    o = ph.photon_bb_stable(dt, kbb, 2048, check=False, out=o)
b.record()
torch.cuda.synchronize()
print(f"cfg {cfg}: A5 {a.elapsed_time(b) / reps:.3f} ms over {int(dt.n_records)} records")
