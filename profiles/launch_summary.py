"""Summarise an ncu --csv launch list: per kernel, launches, mean us, mean DRAM MB read / written."""
import csv, sys

for f in sys.argv[1:]:
    rows = [r for r in csv.reader(open(f)) if len(r) > 10]
    h = rows[0]
    agg = {}
    for r in rows[1:]:
        name = r[h.index("Kernel Name")].split("(")[0].split("::")[-1]
        m = r[h.index("Metric Name")]
        v = float(r[h.index("Metric Value")].replace(",", ""))
        agg.setdefault(name, {}).setdefault(m, []).append(v)
    print("==", f)
    tot = 0.0
    for n, d in agg.items():
        t = d.get("gpu__time_duration.sum", [0]); rd = d.get("dram__bytes_read.sum", [0]); wr = d.get("dram__bytes_write.sum", [0])
        tot += sum(t)
        print(f"{n:28s} n={len(t):3d} us/launch {sum(t)/len(t)/1e3:9.1f}  MB r/w {sum(rd)/len(rd)/1e6:8.1f} {sum(wr)/len(wr)/1e6:8.1f}")
    print(f"total us {tot/1e3:.1f}")
