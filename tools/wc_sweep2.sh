#!/bin/bash
# WC tuning sweep: sub-threads per lane (BK_WC_SUB) x lane bytes x ring depth (ZC gather, 8 MiB window).
mkdir -p gpurun_out
for sub in 4 8 2; do
  for cfg in "4 256" "4 128" "3 256" "4 512" "2 256"; do
    set -- $cfg
    BK_WC_SUB=$sub timeout 300 python bench.py --workload wordcount --gather zc --slots $1 --lane-bytes $2 --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/wc2_${sub}_$1_$2.json 2>gpurun_out/wc2.err
    python3 -c "import json;d=json.load(open('gpurun_out/wc2_${sub}_$1_$2.json'));s=d['stages_ms_per_step'];print('sub=$sub slots=$1 lane=$2', d['value'], d['ms_per_step'], d['config']['n_chunks'], d['config']['lanes_per_chunk'], s['ms_gather'], s['ms_compute'], s['ms_device'], d['link']['frac'])" || tail -3 gpurun_out/wc2.err
  done
done
