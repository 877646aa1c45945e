#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for so in build/variants/*.so; do
  v=$(basename $so .so); [ "$v" = base ] && continue
  HIRACE_LIB=$PWD/$so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "not full and not cfg5" > $OUT/pytest_$v.log 2>&1
  echo "pytest exit $?" >> $OUT/pytest_$v.log
done
REPS=1 CFGS="5 2" timeout 2400 bash scripts/ab4.sh > /dev/null 2>&1
cp $OUT/ab_summary.txt $OUT/ab_summary_occ5.txt
