#!/bin/bash
mkdir -p gpurun_out
for cfg in "dense 4 0" "zc 4 0" "zc 4 256" "zc 8 256" "dense 2 0" "zc 2 512" "zc 4 1024"; do
  set -- $cfg
  timeout 300 python bench.py --workload wordcount --gather $1 --slots $2 --lane-bytes $3 --steps 3 --warmup 2 --no-cpu-baseline > gpurun_out/wc_$1_$2_$3.json 2>gpurun_out/wc.err
  python3 -c "import json;d=json.load(open('gpurun_out/wc_$1_$2_$3.json'));print('$cfg', d['value'], d['ms_per_step'], d['config']['n_chunks'], d['config']['lanes_per_chunk'], d['stages_ms_per_step']['ms_compute'])" || tail -3 gpurun_out/wc.err
done
