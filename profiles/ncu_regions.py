"""Bucket an ncu source page (one kernel) into named line ranges: instruction and stall-sample shares."""
import csv
import io
import subprocess
import sys


def main(rep, fname, regions, n_units):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    agg, cur = {}, None
    for r in csv.reader(io.StringIO(out)):
        if not r:
            continue
        if r[0] == "File Path":
            cur = r[1].split("/")[-1]
            continue
        try:
            line, inst, smp = int(r[0]), int(r[7]), int(r[4])
        except (ValueError, IndexError):
            continue
        key = ("other: " + cur) if cur != fname else next((n for a, b, n in regions if a <= line < b), "other")
        v = agg.setdefault(key, [0, 0])
        v[0] += inst
        v[1] += smp
    ti = sum(v[0] for v in agg.values()) or 1
    ts = sum(v[1] for v in agg.values()) or 1
    for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"{v[0] / ti * 100:5.1f}% inst {v[1] / ts * 100:5.1f}% stall-samples  "
              f"{v[0] * 32 / n_units:6.2f} thread-inst/unit  {k}")


if __name__ == "__main__":
    rep, fname, n_units = sys.argv[1], sys.argv[2], float(sys.argv[3])
    regions = []
    for spec in sys.argv[4:]:  # name:start-end
        n, ab = spec.rsplit(":", 1)
        a, b = ab.split("-")
        regions.append((int(a), int(b), n))
    main(rep, fname, regions, n_units)
