#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { cat $OUT/build.log; exit 1; }
( time timeout 3000 python -m pytest tests -m gpu -q -x --durations=25 ) > $OUT/pytest_gpu_all.log 2>&1; echo "pytest rc=$?"
tail -40 $OUT/pytest_gpu_all.log
