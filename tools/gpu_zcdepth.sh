#!/bin/bash
mkdir -p gpurun_out
for cfg in "4 1" "4 2" "4 3" "5 2" "6 2" "6 3" "3 2"; do set -- $cfg
  BK_ZC_DEPTH=$2 timeout 600 python bench.py --slots $1 --steps 4 --warmup 3 --no-cpu-baseline --no-dbuf --no-profile > gpurun_out/zcd_$1_$2.json 2>gpurun_out/zcd.err
  python3 -c "import json;d=json.load(open('gpurun_out/zcd_$1_$2.json'));print('slots=$1 depth=$2', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'], d['config']['n_chunks'])" || tail -3 gpurun_out/zcd.err
done
