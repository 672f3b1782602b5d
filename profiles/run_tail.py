"""Probe (not the benchmark): fused K1 passes on a config with an instrumented library (abvar/libphoton_tail.so, a
throwaway build whose workers record their start / end globaltimer) -> the spread of the workers' end times."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import tracegen as tg  # noqa: E402
from paper_conf_micro_liusc23_b200 import DeviceTrace, Photon, _lib  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 5
ph = Photon(0)
d = DeviceTrace.from_host(tg.Generator(cfg).trace(), ph.device)
for _ in range(3):
    ph.photon_warp_group(d, None, check=False)
torch.cuda.synchronize()
buf = (ctypes.c_ulonglong * (2 * 4096))()
assert _lib.load().probe_tail_read(buf) == 0
a = np.frombuffer(buf, dtype=np.uint64).reshape(2, 4096).astype(np.int64)
n = int((a[1] > 0).sum())
t0 = a[0, :n].min()
e = np.sort(a[1, :n] - t0) / 1e3
print(f"cfg {cfg} workers {n} end us: min {e[0]:.1f} p10 {e[n // 10]:.1f} p50 {e[n // 2]:.1f} p90 {e[9 * n // 10]:.1f} "
      f"p99 {e[99 * n // 100]:.1f} max {e[-1]:.1f}")
# per-SM view (static mapping: worker gw on CTA gw // 20; interleaved: gw % gridDim)
mode = os.environ.get("TAIL_MAP", "static")
ends = a[1, :n] - t0
sm = (np.arange(n) // 20) if mode == "static" else (np.arange(n) % 148)
per_sm_mean = np.array([ends[sm == s].mean() for s in range(148)]) / 1e3
per_sm_max = np.array([ends[sm == s].max() for s in range(148)]) / 1e3
within = np.array([ends[sm == s].std() for s in range(148)]) / 1e3
print(f"per-SM mean end us: min {per_sm_mean.min():.1f} max {per_sm_mean.max():.1f}; per-SM max end: min "
      f"{per_sm_max.min():.1f} max {per_sm_max.max():.1f}; within-SM std mean {within.mean():.1f}")
order = np.argsort(per_sm_mean)
print("slowest SMs", order[-8:].tolist(), "fastest", order[:8].tolist())
