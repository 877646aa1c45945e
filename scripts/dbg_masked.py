import sys
sys.path.insert(0, '.')
import tracegen as tg, oracle
import paper_conf_sc_jacobsonbg24_b200 as hr
t = tg.random_tiny_masked(0)
print(t.n, len(t.warp_syncs), t.warp_size, t.block_threads, t.grid_blocks)
c = hr.Checker.for_trace(t)
print("set ok")
c.replay(hr.events_to_device(t.events, "cuda:0"))
print(hr.races_to_dict(c.collect()), oracle.races_masked_dict(t))
