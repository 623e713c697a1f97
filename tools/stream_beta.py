import sys, json
sys.path.insert(0,'.')
import torch, tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
def timeit(fn, flush, reps=5):
    ts=[]
    for i in range(reps+2):
        flush.zero_(); e0,e1=torch.cuda.Event(enable_timing=True),torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); e1.synchronize()
        if i>=2: ts.append(e0.elapsed_time(e1))
    return sorted(ts)[len(ts)//2]
flush=torch.empty(256<<20,dtype=torch.uint8,device='cuda')
for c in tcinputs.tccg48()[:8]:
    for dt,tdt in (('f64',torch.float64),('f32',torch.float32)):
        ps=tc.plan(c.expr,c.extents,dt); pg=tc.plan(c.expr,c.extents,dt,stream=False)
        A=tcinputs.uniform(ps.numel('A'),1,device='cuda').to(tdt); B=tcinputs.uniform(ps.numel('B'),2,device='cuda').to(tdt); C=torch.zeros(ps.numel('C'),dtype=tdt,device='cuda')
        print(json.dumps({'id':c.id,'dt':dt,'active':ps.info()['stream'].get('active'),'stream_b1':round(timeit(lambda: ps.execute(A,B,C,beta=1.0),flush),4),'tile_b1':round(timeit(lambda: pg.execute(A,B,C,beta=1.0),flush),4),'stream_b0':round(timeit(lambda: ps.execute(A,B,C),flush),4)}),flush=True)
