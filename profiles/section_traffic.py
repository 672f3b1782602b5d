"""Aggregate the per-section ncu launch lists of profiles/run_section.py into one JSON (DRAM bytes and kernel time
per call of each section), read by bench.py as the `traffic` of its lines:
  python profiles/section_traffic.py OUT.json sec1=gpurun_out/sec_sec1.csv ..."""
import csv
import json
import subprocess
import sys


def one(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    h = rows[0]
    tot = {"dram_bytes": 0.0, "kernel_us": 0.0, "launches": 0, "kernels": {}}
    ids = set()
    for r in rows[1:]:
        m, v = r[h.index("Metric Name")], float(r[h.index("Metric Value")].replace(",", ""))
        name = r[h.index("Kernel Name")].split("(")[0].split("::")[-1]
        ids.add(r[h.index("ID")])
        k = tot["kernels"].setdefault(name, {"dram_bytes": 0.0, "us": 0.0})
        if m.startswith("dram__bytes"):
            tot["dram_bytes"] += v
            k["dram_bytes"] += v
        elif m == "gpu__time_duration.sum":
            tot["kernel_us"] += v / 1e3
            k["us"] += v / 1e3
    tot["launches"] = len(ids)
    return tot


out = {"source": "ncu --profile-from-start off (one call per section, cold-cache serialised launches), "
                 "profiles/run_section.py", "commit": subprocess.run(["git", "rev-parse", "--short", "HEAD"],
                                                                      capture_output=True, text=True).stdout.strip()}
for a in sys.argv[2:]:
    name, path = a.split("=", 1)
    out[name] = one(path)
json.dump(out, open(sys.argv[1], "w"), indent=1)
print(json.dumps({k: (v["dram_bytes"], v["kernel_us"]) if isinstance(v, dict) else v for k, v in out.items()}))
