#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
rm -f $OUT/compact_r2.txt
for cfg in 2 3 4; do for cm in "" "--compact"; do
  timeout 600 python bench.py --config $cfg --steps 20 --warmup 3 --no-per-config --no-slowdown --no-cpu-baseline --no-e2e $cm > $OUT/bc.json 2>/dev/null
  python -c "import json; d=json.loads(open('$OUT/bc.json').read().strip().splitlines()[-1]); print('cfg$cfg', '${cm:-8B}', round(d['value']/1e9,2), 'G acc/s', round(d['ms_per_step'],4), 'ms', d['roofline']['frac'])" >> $OUT/compact_r2.txt
done; done
timeout 900 ncu --set full --clock-control none -k regex:k_tiled -s 1 -c 1 -o $OUT/prof_tiled_inline -f python -c "
import torch, tracegen as tg, paper_conf_sc_jacobsonbg24_b200 as hr
from paper_conf_sc_jacobsonbg24_b200 import examples as ex
t = tg.tiled_reduce(4096, 256, 8, 4, 'half_mask')
c = hr.Checker(t.grid_blocks, t.block_threads, t.warp_size, t.global_words, t.smem_words)
o = torch.zeros(t.global_words, device='cuda')
for _ in range(2):
    c.reset(); ex.tiled(c, o, 4096, 256, 8, 4, 'half_mask', 2 * 4096 * 256)
torch.cuda.synchronize()
" > $OUT/ncu_tiled.log 2>&1
