"""Write profiles/k1_traffic.json (bench.py's roofline "traffic") from an ncu --set full capture of the fused K1:
per-launch dram__bytes_read.sum + dram__bytes_write.sum of the k_bbv3 launch that did the work.
usage: python profiles/k1_traffic_from_ncu.py REPORT.ncu-rep CONFIG [NOTE]"""
import csv
import io
import json
import os
import subprocess
import sys


def main(rep, cfg, note=""):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, data = rows[0], rows[2:]
    best = None
    for r in data:
        name = r[h.index("Kernel Name")]
        if "k_bbv3" not in name:
            continue
        rd = float(r[h.index("dram__bytes_read.sum")].replace(",", ""))
        wr = float(r[h.index("dram__bytes_write.sum")].replace(",", ""))
        unit_r, unit_w = rows[1][h.index("dram__bytes_read.sum")], rows[1][h.index("dram__bytes_write.sum")]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        tot = rd * scale[unit_r] + wr * scale[unit_w]
        if best is None or tot > best[0]:
            best = (tot, name, rd * scale[unit_r], wr * scale[unit_w])
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "k1_traffic.json")
    j = json.load(open(path)) if os.path.exists(path) else {}
    j[str(cfg)] = best[0]
    j[f"{cfg}_detail"] = {"kernel": best[1], "dram_read": best[2], "dram_write": best[3], "capture": note}
    json.dump(j, open(path, "w"), indent=1)
    print(json.dumps(j, indent=1))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else "")
