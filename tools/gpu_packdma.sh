#!/bin/bash
# EXPERIMENT: per-grab DMAs from the packing threads (BK_PACK_DMA) in grep HYBRID / CPU.
mkdir -p gpurun_out
TAG=${TAG:-r01pd}
BK_PACK_DMA=1 timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "grep_medium or grep_adversarial or groupby" -p no:cacheprovider 2>&1 | tail -1
for v in 0 1 4096 65536; do
  for g in hybrid cpu; do
    BK_PACK_DMA=$v timeout 300 python bench.py --steps 5 --warmup 3 --gather $g --no-cpu-baseline --no-dbuf > gpurun_out/${TAG}_${v}_${g}.json 2>/dev/null
    python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_${v}_${g}.json'));print('$v $g', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'], d['stages_ms_per_step']['ms_cpu_gather'], d['stages_ms_per_step']['ms_h2d'])" || echo "$v $g failed"
  done
done
