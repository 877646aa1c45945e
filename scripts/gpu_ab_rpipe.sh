#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build_rp.log 2>&1
for v in rpipe; do
  HIRACE_LIB=$PWD/build/variants/$v.so timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_compact.py -x -q -k "not full and not cfg5" > $OUT/pytest_$v.log 2>&1
  echo "pytest exit $?" >> $OUT/pytest_$v.log
done
CFGS="2 4 3" timeout 1800 bash scripts/ab4.sh
