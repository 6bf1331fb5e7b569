#!/bin/bash
# GPU suite file by file (verbose, per-file timeout) to locate failures / hangs
mkdir -p gpurun_out
T=${TAG:-r02n}
for f in tests/test_gpu_*.py; do
  b=$(basename $f .py)
  timeout 900 python -m pytest $f -v -x --timeout 300 --tb=short -p no:cacheprovider > gpurun_out/${T}_$b.log 2>&1
  echo "$b rc=$? $(grep -cE 'PASSED' gpurun_out/${T}_$b.log) passed; $(grep -E 'FAILED|Timeout' gpurun_out/${T}_$b.log | head -3)"
done
