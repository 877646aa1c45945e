#!/bin/bash
# Generic A/B of build/variants/*.so: parity of every non-base variant (CPU-free GPU subset),
# then kernel time per config (scripts/ab4.sh).  usage: CFGS="2 4" bash scripts/gpu_ab.sh
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for so in build/variants/*.so; do
  v=$(basename $so .so); [ "$v" = base ] && continue
  HIRACE_LIB=$PWD/$so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "not full and not cfg5" > $OUT/pytest_$v.log 2>&1
  echo "pytest exit $?" >> $OUT/pytest_$v.log
done
CFGS=${CFGS:-"2 4"} timeout 1800 bash scripts/ab4.sh
