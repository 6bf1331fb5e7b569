#!/bin/bash
mkdir -p gpurun_out
python -m pytest tests -m gpu -x -q 2>&1 | tail -2
python tools/wc_overhead.py 4
for cfg in "4 256" "6 256" "8 256" "8 512" "3 256"; do set -- $cfg
  timeout 300 python bench.py --workload wordcount --gather zc --slots $1 --lane-bytes $2 --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/wc5_$1_$2.json 2>gpurun_out/wc5.err
  python3 -c "import json;d=json.load(open('gpurun_out/wc5_$1_$2.json'));s=d['stages_ms_per_step'];print('slots=$1 lane=$2', d['value'], d['ms_per_step'], d['config']['n_chunks'], s['ms_h2d'], s['ms_addrgen'], s['ms_gather'], s['ms_compute'], s['ms_device'], d['link']['frac'], d['e2e']['value'], d['overlap']['overlap_frac'])" || tail -3 gpurun_out/wc5.err
done
