"""CPU oracle throughput on C1-C4 (whole configs) and a C5 kernel prefix, for BASELINE.md's table (run on the GPU
box's host; the oracle as it stands, 1 core and all cores): python profiles/cpu_configs.py > out.json"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import tracegen as tg  # noqa: E402

cores = len(os.sched_getaffinity(0))
out = {"cores": cores}
for cfg, k1 in ((1, None), (2, None), (3, None), (4, None), (5, 3000)):
    g = tg.Generator(cfg)
    tr = g.kernels_trace(0, k1 or g.n_kernels)
    t0 = time.perf_counter()
    oracle.analyse(tr)
    d1 = time.perf_counter() - t0
    t0 = time.perf_counter()
    oracle.analyse_threads(tr, cores)
    dn = time.perf_counter() - t0
    out[f"C{cfg}"] = {"events": int(tr.n_events), "kernels": int(tr.n_kernels), "one_core_events_per_s": tr.n_events / d1,
                      "all_cores_events_per_s": tr.n_events / dn, "s_one": d1, "s_all": dn}
    print(cfg, out[f"C{cfg}"], file=sys.stderr, flush=True)
print(json.dumps(out))
