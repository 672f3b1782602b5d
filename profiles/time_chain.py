"""A/B timing probe (not the benchmark): the A1-A4 chain on one config as a CUDA-graph replay (as bench.py times
it) plus the eager per-section times (photon_profile), e.g. PHOTON_LIB_OVERRIDE=abvar/libphoton_X.so."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tracegen as tg  # noqa: E402
from paper_conf_micro_liusc23_b200 import DeviceTrace, Photon  # noqa: E402
from paper_conf_micro_liusc23_b200 import _lib  # noqa: E402
from paper_conf_micro_liusc23_b200._lib import PROF_SECTIONS  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 5
n = int(sys.argv[2]) if len(sys.argv) > 2 else 50
ph = Photon(0)
g = tg.Generator(cfg)
d = DeviceTrace.from_host(g.trace(), ph.device)
L = _lib.load()
r0 = ph.analyse(d, check=True)
graph, r1 = ph.capture(lambda: ph.analyse(d, check=False, out=r0))
for _ in range(3):
    graph.replay()
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(n):
    graph.replay()
b.record()
torch.cuda.synchronize()
ms = a.elapsed_time(b) / n
L.photon_profile(ph.ctx, 1)
for _ in range(n):
    ph.analyse(d, check=False, out=r0)
torch.cuda.synchronize()
pms = (ctypes.c_double * 16)()
pcnt = (ctypes.c_uint64 * 16)()
L.photon_profile_read(ph.ctx, ph.stream_ptr(), pms, pcnt)
L.photon_profile(ph.ctx, 0)
ph.check(r1["_ws"])
ph.check(r1["_mws"])
sec = " ".join(f"{PROF_SECTIONS[i]} {pms[i] / n * 1e3:.0f}" for i in range(len(PROF_SECTIONS)) if pcnt[i])
print(f"cfg {cfg}: graph {ms:.4f} ms | eager us: {sec}")
