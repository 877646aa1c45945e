#!/bin/bash
# Tail-pool A/B: parity of the variants, then bench cfg2/3/4 per variant (scripts/ab4.sh).
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_tail.log 2>&1
for v in tail1 tail2 tail3; do
  HIRACE_LIB=$PWD/build/variants/$v.so timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_compact.py -x -q -k "not full and not cfg5" > $OUT/pytest_$v.log 2>&1
  echo "pytest exit $?" >> $OUT/pytest_$v.log
done
CFGS="2 4 3" timeout 1800 bash scripts/ab4.sh
