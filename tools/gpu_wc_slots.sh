#!/bin/bash
# Word count (C1: 64 MiB, 8 MiB window): ring depth sweep on the current code.
mkdir -p gpurun_out
TAG=${TAG:-r01w}
for sl in ${SLOTS:-6 8 10 12 16}; do
  for rep in 1 2; do
    timeout 300 python bench.py --workload wordcount --steps 30 --warmup 5 --slots $sl --no-cpu-baseline --no-dbuf $ARGS > gpurun_out/${TAG}_wc_${sl}_${rep}.json 2>/dev/null
    python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_wc_${sl}_${rep}.json'));print($sl, d['value'], d['ms_per_step'], d['config']['n_chunks'], d['config']['chunk_budget_bytes'])" || echo "$sl failed"
  done
done
