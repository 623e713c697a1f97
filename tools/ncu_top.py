"""Summaries of an ncu report: key raw metrics and the SASS lines with the most stall samples.
usage: python tools/ncu_top.py report.ncu-rep [ntop]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 25
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
h, u, v = r[0], r[1], r[2]
keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum",
        "sm__cycles_elapsed.avg", "smsp__cycles_active.avg", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "lts__t_sectors_srcunit_tex_op_read.sum",
        "lts__t_sectors_srcunit_tex_op_write.sum", "launch__registers_per_thread", "launch__grid_size",
        "sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_uniform.avg.pct_of_peak_sustained_active"]
for k in keys:
    if k in h:
        print(f"{k:70s} {u[h.index(k)]:>10s} {v[h.index(k)]}")
for i, n in enumerate(h):
    if n.startswith("smsp__average_warps_issue_stalled_") and n.endswith("_per_issue_active.ratio"):
        try:
            if float(v[i]) > 0.1:
                print(f"  stall {n[34:-23]:28s} {v[i]}")
        except ValueError:
            pass
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(src)))
h = r[1]
rows = [x for x in r[2:] if len(x) == len(h) and x[0] != h[0]]
ia, isrc = h.index("Address"), h.index("Source")
iss, iex = h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
def num(v):
    try:
        return float(v or 0)
    except ValueError:
        return 0.0


rows = [x for x in rows if num(x[iss]) or num(x[iex])]
tot = sum(num(x[iss]) for x in rows)
print("stall samples", tot)
for x in sorted(rows, key=lambda x: -num(x[iss]))[:ntop]:
    print(f"  {int(x[ia], 16) & 0xffff:#06x} {x[isrc][:70]:70s} {x[iss]:>7s} {x[iex]}")
