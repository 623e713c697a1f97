"""Stall samples and executions aggregated by SASS opcode (and by code region) from an ncu
report's source page.  usage: python tools/ncu_ops.py report.ncu-rep"""
import collections
import csv
import io
import subprocess
import sys

src = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "sass"],
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


by = collections.defaultdict(lambda: [0.0, 0.0])
for x in rows:
    s = x[isrc].split()
    if not s:
        continue
    op = s[1] if s[0].startswith("@") and len(s) > 1 else s[0]
    op = op.split(".")[0]
    by[op][0] += num(x[iss])
    by[op][1] += num(x[iex])
tot = sum(v[0] for v in by.values())
for op, (st, ex) in sorted(by.items(), key=lambda kv: -kv[1][0])[:25]:
    print(f"{op:12s} stall {st:9.0f} ({100 * st / tot:5.1f}%)  executed {ex:12.0f}")
