import sys, os, time
sys.path.insert(0, os.getcwd())
import torch, numpy as np
import paper_conf_sc_jacobsonbg24_b200 as hr, tracegen as tg
t = tg.cfg2(True)
c = hr.Checker.for_trace(t)
d = hr.events_to_device(t.events)
cap = 1 << 20
out = torch.empty(cap * 16, dtype=torch.uint8, device="cuda")
tot = torch.zeros(1, dtype=torch.int64, device="cuda")
s = torch.cuda.Stream()
torch.cuda.synchronize()
def step():
    c.reset(s)
    c.check_device(d, out, cap, tot, stream=s)
for _ in range(5):
    step()
torch.cuda.synchronize()
K = 200
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(s)
for _ in range(K):
    step()
e1.record(s)
torch.cuda.synchronize()
print("eager ms/step", e0.elapsed_time(e1) / K, "flagged", int(tot.item()))
g = torch.cuda.CUDAGraph()
try:
    with torch.cuda.graph(g, stream=s):
        step()
    tot.zero_()
    with torch.cuda.stream(s):
        for _ in range(5):
            g.replay()
    torch.cuda.synchronize()
    print("after graph replays flagged", int(tot.item()))
    e0.record(s)
    with torch.cuda.stream(s):
        for _ in range(K):
            g.replay()
    e1.record(s)
    torch.cuda.synchronize()
    print("graph ms/step", e0.elapsed_time(e1) / K, "flagged", int(tot.item()), "sync", c.sync())
except Exception as ex:
    print("graph failed", repr(ex))
