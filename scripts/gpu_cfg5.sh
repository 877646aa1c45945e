#!/bin/bash
# config 5 on one GPU: parity (medium + full 1e9), bench N=1, and a 2-rank sharded run on the one GPU (gloo host staging)
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
nproc > $OUT/cfg5_env.txt; free -g >> $OUT/cfg5_env.txt
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -k "cfg5" > $OUT/pytest_cfg5.log 2>&1
timeout 900 python bench.py --config 5 --steps 5 --warmup 3 --no-cpu-baseline > $OUT/bench_c5.json 2> $OUT/bench_c5.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29531 \
   bench.py --gpus 2 --config 5 --steps 3 --warmup 3 --transport host > $OUT/bench_c5_p2host.json 2> $OUT/bench_c5_p2host.err
