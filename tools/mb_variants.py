import sys, json, os
sys.path.insert(0, "/root/repo")
import torch, tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
HBM = 6547.8e9
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
def timeit(p, A, B, C, reps=5):
    ts = []
    for i in range(reps + 2):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); p.execute(A, B, C); e1.record(); e1.synchronize()
        if i >= 2: ts.append(e0.elapsed_time(e1))
    return sorted(ts)[len(ts) // 2]
for c in [c for c in tcinputs.tccg48() if c.id <= 8]:
    p0 = tc.plan(c.expr, c.extents)
    A = tcinputs.uniform(p0.numel("A"), 1000 + c.id, device="cuda")
    B = tcinputs.uniform(p0.numel("B"), 2000 + c.id, device="cuda")
    C = torch.empty(p0.numel("C"), dtype=torch.float64, device="cuda")
    byts = 8 * (p0.numel("A") + p0.numel("B") + p0.numel("C"))
    row = {"id": c.id}
    for v in (None, 8, 17, 25, 26):
        for mo in (None, "X"):
            try:
                p = tc.plan(c.expr, c.extents, variant=v, morder=mo)
                ms = timeit(p, A, B, C)
                row[f"{v}{mo or ''}"] = round(byts / (ms * 1e-3) / HBM, 3)
            except Exception as e:
                row[f"{v}{mo or ''}"] = str(e)[:30]
    pt = tc.plan(c.expr, c.extents).tuned(A, B, C, topk=8, reps=2)
    row["tuned"] = round(byts / (timeit(pt, A, B, C) * 1e-3) / HBM, 3); row["tuned_v"] = pt.info()["variant"]
    print(json.dumps(row), flush=True)
