#!/bin/bash
# host assembly sweep on the GPU box's host (prefetch distance x tiles per grab), then grep bench with the best guesses
mkdir -p gpurun_out
nproc; lscpu | grep -E "Model name|Thread|Core|Socket|NUMA" | head -6
for cfg in "16 16" "0 16" "32 16" "64 16" "32 64" "64 64" "128 64"; do set -- $cfg
  echo "pf=$1 grab=$2"; BK_HG_PF=$1 BK_HG_GRAB=$2 timeout 300 ./build/hgb 16 16 | tail -1
done
for cfg in "16 16" "32 16" "64 64"; do set -- $cfg
  BK_HG_PF=$1 BK_HG_GRAB=$2 timeout 600 python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-dbuf --no-profile > gpurun_out/hg_$1_$2.json 2>gpurun_out/hg.err
  python3 -c "import json;d=json.load(open('gpurun_out/hg_$1_$2.json'));print('bench pf=$1 grab=$2', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'])" || tail -3 gpurun_out/hg.err
done
