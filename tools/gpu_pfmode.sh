#!/bin/bash
# EXPERIMENT: software-prefetch flavour of the host packers (BK_PF_MODE: 0 t0, 1 nta, 2 t2, 3 nta x2 lines).
mkdir -p gpurun_out
TAG=${TAG:-r01pf}
for m in 0 1 2 3; do echo "pack alone mode $m: $(BK_PF_MODE=$m ./build/hgb 16 16 pack | tail -1)"; done
for m in 0 1 3 0 1 3; do
  for g in hybrid cpu; do
    BK_PF_MODE=$m timeout 300 python bench.py --steps 5 --warmup 3 --gather $g --no-cpu-baseline --no-dbuf > gpurun_out/${TAG}_${m}_${g}.json 2>/dev/null
    python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_${m}_${g}.json'));print('mode $m $g', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'], d['stages_ms_per_step']['ms_cpu_gather'])" || echo "$m $g failed"
  done
done
