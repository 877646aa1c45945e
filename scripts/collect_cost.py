import sys, os
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_sc_jacobsonbg24_b200 as hr, tracegen as tg
t = tg.cfg2(True)
c = hr.Checker.for_trace(t)
d = hr.events_to_device(t.events)
cap = 1 << 20
out = torch.empty(cap * 16, dtype=torch.uint8, device="cuda")
tot = torch.zeros(1, dtype=torch.int64, device="cuda")
s = torch.cuda.current_stream()
K = 100
a = [torch.cuda.Event(enable_timing=True) for _ in range(K)]
b = [torch.cuda.Event(enable_timing=True) for _ in range(K)]
for e in a + b: e.record()
def run(fused):
    tt = 0.0
    for i in range(K + 5):
        c.reset()
        if i >= 5: c.set_kernel_timing(a[i-5], b[i-5])
        else: c.set_kernel_timing(None, None)
        if fused: c.check_device(d, out, cap, tot)
        else: c.replay(d)
    torch.cuda.synchronize()
    c.set_kernel_timing(None, None)
    return sum(x.elapsed_time(y) for x, y in zip(a, b)) / K
print("replay only ms", run(False))
print("replay + fused collect ms", run(True))

# standalone collect kernel after a replay-only kernel
ca = torch.cuda.Event(enable_timing=True); cb = torch.cuda.Event(enable_timing=True)
tot_ms = 0.0
for i in range(K + 5):
    c.reset()
    c.replay(d)
    ca.record()
    c.collect_device(out, cap, tot)
    cb.record()
    torch.cuda.synchronize()
    if i >= 5:
        tot_ms += ca.elapsed_time(cb)
print("standalone collect ms", tot_ms / K, "flagged", int(tot.item()))
