#!/bin/bash
# compute-sanitizer memcheck over smoke() (every path the driver smokes: batch-major 8-byte and
# compact records, window-major, cluster) and a medium config-5 window check.
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { cat $OUT/build.log; exit 1; }
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/memcheck_smoke.log 2>&1
echo "smoke memcheck rc=$?"; tail -3 $OUT/memcheck_smoke.log
WL=12 REPS=2 BLOCKS=1024 WORDS_LOG2=26 timeout 600 compute-sanitizer --tool memcheck --print-limit 20 python scripts/prof_window.py > $OUT/memcheck_window.log 2>&1
echo "window memcheck rc=$?"; tail -3 $OUT/memcheck_window.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()"
