"""Text summary of one ncu report (key throughput metrics, DRAM bytes, stall mix, the hottest
SASS lines) for profiles/.  usage: python tools/ncu_summary.py report.ncu-rep [title]"""
import collections
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed", "sm__inst_executed_pipe_tma.avg.pct_of_peak_sustained_active",
        "l1tex__m_xbar2l1tex_read_bytes.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "smsp__sass_inst_executed_op_tma_ld.sum"]


def page(rep, *args):
    out = subprocess.run(["ncu", "-i", rep, "--csv"] + list(args), capture_output=True, text=True).stdout
    return list(csv.reader(io.StringIO(out)))


def main():
    rep = sys.argv[1]
    title = sys.argv[2] if len(sys.argv) > 2 else rep
    raw = page(rep, "--page", "raw")
    d = dict(zip(raw[0], raw[2]))
    print(f"# {title}\n# {d.get('Kernel Name', '')[:160]}")
    for k in KEYS:
        if k in d:
            print(f"{k:70s} {d[k]} {raw[1][raw[0].index(k)]}")
    src = page(rep, "--page", "source", "--print-source", "sass")
    h, rows = src[1], src[2:]
    iw = h.index("Warp Stall Sampling (All Samples)")
    reasons = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
    tot = collections.Counter()
    for x in rows:
        for c in reasons:
            tot[c] += float(x[h.index(c)] or 0)
    s = sum(tot.values()) or 1
    print("stall mix:", ", ".join(f"{c[6:]} {n / s:.2f}" for c, n in tot.most_common(8)))
    print("hottest SASS (samples, executions):")
    ia, isrc, ie = h.index("Address"), h.index("Source"), h.index("Instructions Executed")
    for x in sorted(rows, key=lambda x: -float(x[iw] or 0))[:12]:
        print(f"  {x[ia][-5:]} {x[isrc][:80]:80s} {x[iw]:>6s} {x[ie]}")


if __name__ == "__main__":
    main()
