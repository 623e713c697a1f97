"""Registers / spills per FP64 kernel instance from `nvcc -Xptxas -v` output on stdin."""
import re
import sys

cur = None
for line in sys.stdin:
    m = re.search(r"Compiling entry function '(\S+)'", line)
    if m:
        k = re.findall(r"ELi(\d+)|Li(\d+)E|Lb([01])", m.group(1))
        nums = [a or b or c for a, b, c in k]
        cur = "x".join(nums[:3]) + " w" + "x".join(nums[3:5]) + " st" + nums[5] + " occ" + nums[7] + " xk/yk/stg " + "".join(nums[8:11]) if "f64" in m.group(1) else m.group(1)[:60]
    m = re.search(r"Used (\d+) registers", line)
    if m and cur:
        regs = m.group(1)
    m2 = re.search(r"(\d+) bytes spill stores, (\d+) bytes spill loads", line)
    if m2 and cur:
        print(f"{cur:50s} spill st {m2.group(1):>5s} ld {m2.group(2):>5s}", end="")
    if m and cur:
        print(f"  regs {regs}")
        cur = None
