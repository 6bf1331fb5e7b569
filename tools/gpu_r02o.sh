#!/bin/bash
mkdir -p gpurun_out
T=${TAG:-r02o}
for f in tests/test_gpu_kmer.py tests/test_gpu_bench_ranks.py tests/test_gpu_ranks_parity.py; do
  b=$(basename $f .py)
  timeout 1200 python -m pytest $f -v --timeout 400 --tb=short -p no:cacheprovider > gpurun_out/${T}_$b.log 2>&1
  echo "$b rc=$? $(grep -cE 'PASSED' gpurun_out/${T}_$b.log) passed; $(grep -E 'FAILED|Timeout' gpurun_out/${T}_$b.log | head -3)"
done
bash tools/gpu_r02m.sh
