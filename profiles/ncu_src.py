"""Per-source-line view of one kernel in an ncu report (needs -lineinfo and --import-source): warp / thread
instructions, shared-memory wavefronts (actual and ideal) and the dominant stall reasons of each line.
usage: python profiles/ncu_src.py REPORT.ncu-rep FILE.cu N_UNITS [TOP]   (N_UNITS = events per launch, for ratios)"""
import csv
import io
import subprocess
import sys


def main(rep, fname, n_units, top=40):
    import os
    kf = ["-k", "regex:" + os.environ["KFILTER"]] if os.environ.get("KFILTER") else []  # one kernel of a report
    out = subprocess.run(["ncu", "-i", rep] + kf + ["--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, cur, agg = None, None, {}
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            cur = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or cur is None:
            continue
        try:
            line = int(r[0])
        except ValueError:
            continue
        v = agg.setdefault((cur, line), {"src": r[1][:80]})
        for i, name in enumerate(hdr):
            if i < 2:
                continue
            try:
                v[name] = v.get(name, 0) + float(r[i].replace(",", "")) if r[i] else v.get(name, 0)
            except ValueError:
                pass
    ti = sum(v.get("Instructions Executed", 0) for v in agg.values()) or 1
    ts = sum(v.get("Warp Stall Sampling (All Samples)", 0) for v in agg.values()) or 1
    tw = sum(v.get("L1 Wavefronts Shared", 0) for v in agg.values()) or 1
    stalls = [n for n in hdr if n.startswith("stall_") and "Not Issued" not in n] if hdr else []
    print(f"total: {ti / 1e6:.1f}M warp-inst ({ti * 32 / n_units:.1f} thread-slots/unit), "
          f"{tw / 1e6:.1f}M smem wavefronts ({tw * 32 / n_units:.2f} per 32 units), {ts:.0f} samples")
    keys = sorted(agg, key=lambda k: -agg[k].get("Warp Stall Sampling (All Samples)", 0))[:top]
    for k in keys:
        v = agg[k]
        st = sorted(((v.get(n, 0), n[6:]) for n in stalls), reverse=True)[:3]
        sst = sum(v.get(n, 0) for n in stalls) or 1
        print(f"{k[0][:12]:12s}{k[1]:5d} smp {100 * v.get('Warp Stall Sampling (All Samples)', 0) / ts:5.2f}% "
              f"inst {100 * v.get('Instructions Executed', 0) / ti:5.2f}% "
              f"thr/u {v.get('Thread Instructions Executed', 0) / n_units:5.2f} "
              f"wf/32u {v.get('L1 Wavefronts Shared', 0) * 32 / n_units:5.2f} "
              f"({', '.join(f'{n} {100 * c / sst:.0f}%' for c, n in st)})  {v['src']}")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], float(sys.argv[3]), int(sys.argv[4]) if len(sys.argv) > 4 else 40)
