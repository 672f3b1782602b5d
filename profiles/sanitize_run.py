"""Every C-ABI entry point once on small seeded inputs, for compute-sanitizer (tests/test_sanitizer.py):
  compute-sanitizer --tool memcheck --error-exitcode 9 python profiles/sanitize_run.py [all|k1]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import tracegen as tg  # noqa: E402
from paper_conf_micro_liusc23_b200 import DeviceTiming, DeviceTrace, Photon, to_device  # noqa: E402
from paper_conf_micro_liusc23_b200.dist import GpuBackend, ROW_BYTES  # noqa: E402

what = sys.argv[1] if len(sys.argv) > 1 else "all"
ph = Photon(0)
g = tg.Generator(6)
tr = g.trace()
d = DeviceTrace.from_host(tr, ph.device)
o = ph.photon_bbv_build(d, bbv16=True, insts=True, kbb=True)
ty = ph.analyse(d, want_dist=True)  # fused K1, canonicalisation, A3/A4 (two streams)
# the other shared-memory-heavy kernels (racecheck / synccheck run "k1"): A5's byte-counter histograms and window
# ring, N2's verification histograms
ph.photon_bb_stable(DeviceTiming.from_host(g.timing(), ph.device), o["kernel_bb_insts"], 64)
ph.photon_warp_group_full(d, o["warp_bbv16"])
if what == "all":
    ph.photon_warp_group(d, o["warp_bbv16"])  # unfused grouping
    K = tr.n_kernels
    gb = ph.photon_gpu_bbv(K, ty)
    be = GpuBackend(ph)  # the split multi-GPU calls
    rows = torch.zeros((4096, ROW_BYTES), dtype=torch.uint8, device=ph.device)
    n_rows = torch.zeros(1, dtype=torch.int64, device=ph.device)
    ph.photon_types_export(K, ty, 0, 0, rows, n_rows)
    gg = be.alloc_global(K, 4096)
    be.merge(rows, 4096, K, d.warps_total, gg)
    wt = ph.empty(tr.n_warps, "int32")
    be.remap(d, ty, gg, 0, K, wt)
    sig = ph.empty(16 * 4096, "int64")
    mass = ph.empty(K, "int64")
    be.sig_build(gg, K, 0, K, sig, mass)
    pairs = ph.empty(16 * K + 65536, "int64")
    npairs = ph.empty(1, "int64")
    prm = ph.match_params()
    be.match_scan(gg, K, sig, mass, d.warps_total, prm, 0, K, pairs, npairs)
    match, dist = ph.empty(K, "int64"), ph.empty(K, "float64")
    be.match_resolve(gg, K, sig, mass, d.warps_total, prm, pairs, match, dist)
    tm = DeviceTiming.from_host(g.timing(), ph.device)
    st = ph.photon_bb_stable(tm, o["kernel_bb_insts"], 16)
    ph.photon_bb_predict(d, st["first_stable"], st["stable_dur_sum"])
    ph.photon_warp_stable(DeviceTiming.from_host(g.warp_timing(), ph.device), ty["warp_sampling_ok"], 32)
    ph.photon_kernel_predict(ty["match"], gb["mass"], to_device(np.arange(K, dtype=np.uint64) + 100, ph.device),
                             to_device(np.arange(K, dtype=np.uint64) * 7 + 1000, ph.device))
    W = tr.n_warps
    owner = np.repeat(np.arange(W), np.diff(tr.warp_event_off.astype(np.int64))).astype(np.int32)
    ph.photon_ingest_tagged(torch.from_numpy(owner).to(ph.device), torch.from_numpy(tr.bb.view(np.int16)).to(ph.device),
                            W)
    pool = ph.photon_pool_export(K, ty, d.warps_total, ty["match"])
    ph.photon_kernel_match_pooled(pool, K, ty, d.warps_total)
torch.cuda.synchronize()
print("sanitize run ok", what)
