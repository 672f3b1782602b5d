"""Summarise an ncu report: key throughput counters, stall breakdown, top source lines (used for profiles/*.md)."""
import csv
import io
import subprocess
import sys


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def main(rep):
    h, units, data = raw(rep)
    keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
            "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.avg.per_cycle_active",
            "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
            "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "launch__registers_per_thread",
            "launch__occupancy_limit_shared_mem", "launch__grid_size", "sm__cycles_elapsed.avg.per_second"]
    for row in data:
        name = row[h.index("Kernel Name")][:90]
        print(f"== {name}")
        for k in keys:
            if k in h:
                print(f"  {k:75s} {row[h.index(k)]:>16s} {units[h.index(k)]}")
        st = []
        for i, n in enumerate(h):
            if n.startswith("smsp__pcsamp_warps_issue_stalled_") and not n.endswith("not_issued"):
                try:
                    st.append((n.replace("smsp__pcsamp_warps_issue_stalled_", ""), float(row[i].replace(",", ""))))
                except ValueError:
                    pass
        tot = sum(v for _, v in st) or 1
        print("  stalls: " + ", ".join(f"{n} {100 * v / tot:.1f}%" for n, v in sorted(st, key=lambda x: -x[1])[:8]))


if __name__ == "__main__":
    main(sys.argv[1])
