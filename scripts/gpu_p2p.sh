#!/bin/bash
# Peer dispatch + streaming collect round: build, sharded/compact/collect GPU tests, benches,
# and config 5 peer-dispatch sharded over 2 processes sharing the one GPU.
TAG=${1:-p}
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_sharded.py tests/test_gpu_compact.py -x -q > $OUT/pytest_p2p_$TAG.log 2>&1
echo "pytest exit $?" >> $OUT/pytest_p2p_$TAG.log
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "not full and not cfg5" > $OUT/pytest_parity_$TAG.log 2>&1
echo "pytest exit $?" >> $OUT/pytest_parity_$TAG.log
for cfg in 2 3 4; do
  timeout 600 python bench.py --config $cfg --no-cpu-baseline --no-slowdown --no-e2e --steps 50 > $OUT/bench_cfg${cfg}_$TAG.json 2> $OUT/bench_cfg${cfg}_$TAG.err
done
timeout 1500 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29555 \
  bench.py --config 5 --gpus 2 --transport p2p --steps 3 --warmup 3 > $OUT/bench_cfg5_p2p2_$TAG.json 2> $OUT/bench_cfg5_p2p2_$TAG.err
ls -la $OUT | tail -8
