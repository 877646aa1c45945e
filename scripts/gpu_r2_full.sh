#!/bin/bash
# Full GPU suite, smoke and the default bench line on the committed tree.
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { cat $OUT/build.log; exit 1; }
( time timeout 3000 python -m pytest tests -m gpu -q --durations=25 ) > $OUT/pytest_gpu_all.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
( time timeout 1500 python bench.py ) > $OUT/bench_default.json 2> $OUT/bench_default.err
tail -5 $OUT/pytest_gpu_all.log
