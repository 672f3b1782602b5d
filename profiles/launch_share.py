"""Per-kernel share of a step from an ncu launch list (--metrics gpu__time_duration.sum --csv)."""
import collections
import csv
import sys


def main(path):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        v = float(r[vi].replace(",", ""))
        v = v * 1e3 if r[ui] == "usecond" else (v * 1e6 if r[ui] == "msecond" else v)
        name = r[ki].split("(")[0].replace("void ", "").replace("photon::<unnamed>::", "").replace("unnamed>::", "")
        agg[name][0] += 1
        agg[name][1] += v
    tot = sum(v for _, v in agg.values())
    print(f"{'us/launch':>10} {'share':>6} {'n':>4}  kernel   (cold-cache, serialised under ncu: compare shares)")
    for n, (c, v) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"{v / c / 1e3:10.1f} {100 * v / tot:5.1f}% {c:4d}  {n}")


if __name__ == "__main__":
    main(sys.argv[1])
