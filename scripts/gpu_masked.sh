#!/bin/bash
# masked-sync GPU parity (tests/test_gpu_masked.py) + a smoke of the rest
OUT=gpurun_out
mkdir -p $OUT
timeout 1200 python -m pytest tests/test_gpu_masked.py -x -q > $OUT/pytest_masked.log 2>&1
echo "pytest exit $?" >> $OUT/pytest_masked.log
