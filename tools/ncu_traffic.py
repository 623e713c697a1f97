"""profiles/ncu_traffic.json from an `ncu --set full --profile-from-start off` capture of
`bench.py --profile` (one launch per TCCG case, in gpurun_out/profile_cases.json order).
usage: python tools/ncu_traffic.py report.ncu-rep gpurun_out/profile_cases.json out.json"""
import csv
import io
import json
import subprocess
import sys

rep, cases_json, out = sys.argv[1:4]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
h, rows = r[0], r[2:]
ik = h.index("Kernel Name")
get = lambda row, k: float(row[h.index(k)].replace(",", ""))
rows = [x for x in rows if x[ik].startswith("void tc_") or x[ik].startswith("tc_")]
cases = json.load(open(cases_json))
assert len(rows) == len(cases), (len(rows), len(cases))
launches = []
for x, c in zip(rows, cases):
    rd, wr = get(x, "dram__bytes_read.sum"), get(x, "dram__bytes_write.sum")
    # ncu reports bytes with a unit row (r[1]); normalise to bytes
    u = dict(zip(h, r[1]))
    sc = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    rd *= sc.get(u["dram__bytes_read.sum"], 1)
    wr *= sc.get(u["dram__bytes_write.sum"], 1)
    t = get(x, "gpu__time_duration.sum") * {"ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "nsecond": 1e-9,
                                            "ms": 1e-3, "msecond": 1e-3}.get(u["gpu__time_duration.sum"], 1e-9)
    launches.append({"case": c["case"], "kernel": c["kernel"], "dram_bytes": int(rd + wr),
                     "dram_read": int(rd), "dram_write": int(wr), "alg_bytes": c["alg_bytes"],
                     "ncu_time_s": t, "ncu_tflops": c["flops"] / t / 1e12})
json.dump({"how": "ncu --set full --clock-control none --profile-from-start off, bench.py --profile "
                  "(one cold-L2 launch per case)", "launches": launches}, open(out, "w"), indent=1)
print(f"{len(launches)} launches -> {out}")
