#!/bin/bash
mkdir -p gpurun_out
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-dbuf"
for cfg in "4 0" "3 0" "5 0" "4 128" "4 512" "4 1024" "6 0" "4 0"; do
  set -- $cfg
  timeout 600 $B --slots $1 --lane-bytes $2 2>/dev/null | python3 -c "import json,sys;d=json.loads(sys.stdin.read());s=d['stages_ms_per_step'];print('slots=$1 lane=$2', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'], s['ms_compute'])"
done
