"""Per-source-line instruction / stall-sample shares of one kernel in an ncu report (source page, -lineinfo)."""
import csv
import io
import subprocess
import sys


def main(rep, n_units=None, top=40, bucket=0):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    agg, fname, cur = {}, None, None
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r[0] in ("Function Name", "Line No"):
            continue
        if r[0] != "":
            line = int(r[0])
            cur = (fname, line // bucket * bucket if bucket else line, r[1][:100] if not bucket else "")
            agg.setdefault(cur, [0, 0])
            try:
                agg[cur][0] += int(r[7])
                agg[cur][1] += int(r[4])
            except ValueError:
                pass
    ti = sum(v[0] for v in agg.values()) or 1
    ts = sum(v[1] for v in agg.values()) or 1
    print(f"warp instructions {ti}, stall samples {ts}" +
          (f", thread-instructions per unit {ti * 32 / n_units:.2f}" if n_units else ""))
    items = sorted(agg.items(), key=lambda kv: -kv[1][0]) if not bucket else sorted(agg.items())
    for (f, ln, src), (i, s) in items[:top] if not bucket else items:
        if bucket and i / ti < 0.003 and s / ts < 0.003:
            continue
        print(f"{i / ti * 100:5.1f}% inst {s / ts * 100:5.1f}% smp  {f}:{ln}  {src}")


if __name__ == "__main__":
    rep = sys.argv[1]
    n = float(sys.argv[2]) if len(sys.argv) > 2 else None
    b = int(sys.argv[3]) if len(sys.argv) > 3 else 0
    main(rep, n, bucket=b)
