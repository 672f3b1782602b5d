"""Timing probe (not the benchmark): K1 variants on one config -- fused (BBV + tile de-dup), BBV-only (bbv16 out),
insts-only -- with CUDA events, to separate the streaming pass from the grouping epilogue."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tracegen as tg  # noqa: E402
from paper_conf_micro_liusc23_b200 import DeviceTrace, Photon  # noqa: E402
from paper_conf_micro_liusc23_b200 import _lib  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 5
ph = Photon(0)
g = tg.Generator(cfg)
d = DeviceTrace.from_host(g.trace(), ph.device)
L = _lib.load()


def timeit(fn, n=10):
    fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(n):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n


o1 = {}
t_fused = timeit(lambda: ph.photon_warp_group(d, None, check=False))
t_b16 = timeit(lambda: ph.photon_bbv_build(d, bbv16=True, insts=False, check=False, out=o1))
o2 = {}
t_ins = timeit(lambda: ph.photon_bbv_build(d, bbv16=False, insts=True, check=False, out=o2))
E = g.n_events if hasattr(g, "n_events") else int(d.n_events)
print(f"cfg {cfg}: warp_group (fused K1 + canon) {t_fused:.3f} ms | bbv_build bbv16 {t_b16:.3f} ms | "
      f"bbv_build insts {t_ins:.3f} ms | E={E}")
