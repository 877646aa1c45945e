#!/bin/bash
# Report-buffer collect round: build, GPU tests touching collection, bench configs 3 and 5,
# then the occupancy A/B of build/variants (scripts/ab4.sh).
TAG=${1:-r}
OUT=gpurun_out
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_$TAG.log 2>&1
timeout 900 python -m pytest tests/test_gpu_compact.py tests/test_gpu_parity.py -x -q -k "report or collect or cfg3 or cfg5 or fused or compact" > $OUT/pytest_rep_$TAG.log 2>&1
echo "pytest exit $?" >> $OUT/pytest_rep_$TAG.log
timeout 600 python bench.py --config 3 --no-cpu-baseline --no-slowdown --no-e2e --steps 30 > $OUT/bench_cfg3_$TAG.json 2> $OUT/bench_cfg3_$TAG.err
timeout 900 python bench.py --config 5 --no-cpu-baseline --no-slowdown --no-e2e --steps 5 > $OUT/bench_cfg5_$TAG.json 2> $OUT/bench_cfg5_$TAG.err
HIRACE_COLLECT=scan timeout 900 python bench.py --config 5 --no-cpu-baseline --no-slowdown --no-e2e --steps 5 > $OUT/bench_cfg5scan_$TAG.json 2> $OUT/bench_cfg5scan_$TAG.err
CFGS="2 4" timeout 1500 bash scripts/ab4.sh
ls -la $OUT | tail -8
