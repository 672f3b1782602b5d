"""Profiling driver (not a benchmark): one section of bench.py, warmed up, then ONE call inside a
cudaProfilerStart/Stop range, for `ncu --profile-from-start off` (per-kernel DRAM bytes of exactly one call):
  ncu --profile-from-start off --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
      --csv --log-file gpurun_out/sec_a5.csv python profiles/run_section.py a5
sections: chain (C5 A1-A4), a5 (C3), a5_c5 (C5 kernels [0, 1000)), n1, n2, n3 (C3)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tracegen as tg  # noqa: E402
from paper_conf_micro_liusc23_b200 import DeviceTiming, DeviceTrace, Photon  # noqa: E402

sec = sys.argv[1]
ph = Photon(0)
if sec == "chain":
    d = DeviceTrace.from_host(tg.Generator(5).trace(), ph.device)
    r = ph.analyse(d)
    fn = lambda: ph.analyse(d, check=False, out=r)
elif sec in ("a5", "a5_c5", "n3"):
    g = tg.Generator(3 if sec != "a5_c5" else 5)
    k1 = g.n_kernels if sec != "a5_c5" else 1000
    da = DeviceTrace.from_host(g.kernels_trace(0, k1), ph.device)
    kbb = ph.photon_bbv_build(da, bbv16=False, insts=False, kbb=True)["kernel_bb_insts"]
    dt = DeviceTiming.from_host(g.timing(0, k1), ph.device)
    o = ph.photon_bb_stable(dt, kbb, 2048)
    if sec == "n3":
        o3 = ph.photon_bb_predict(da, o["first_stable"], o["stable_dur_sum"])
        fn = lambda: ph.photon_bb_predict(da, o["first_stable"], o["stable_dur_sum"], check=False, out=o3)
    else:
        fn = lambda: ph.photon_bb_stable(dt, kbb, 2048, check=False, out=o)
elif sec == "n1":
    g = tg.Generator(3)
    ok = ph.photon_warp_group(DeviceTrace.from_host(g.trace(), ph.device))["warp_sampling_ok"]
    dw = DeviceTiming.from_host(g.warp_timing(), ph.device)
    o = ph.photon_warp_stable(dw, ok, 1024)
    fn = lambda: ph.photon_warp_stable(dw, ok, 1024, check=False, out=o)
elif sec == "n2":
    g = tg.Generator(3)
    d2 = DeviceTrace.from_host(g.trace(), ph.device)
    b16 = ph.photon_bbv_build(d2, bbv16=True, insts=False)["warp_bbv16"]
    o = ph.photon_warp_group_full(d2, b16)
    fn = lambda: ph.photon_warp_group_full(d2, b16, check=False, out=o)
else:
    raise SystemExit(f"unknown section {sec}")
fn()
torch.cuda.synchronize()
torch.cuda.profiler.start()
fn()
torch.cuda.synchronize()
torch.cuda.profiler.stop()
