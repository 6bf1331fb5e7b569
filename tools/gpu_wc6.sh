#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-r01w2}
python -m pytest tests -m gpu -x -q -k "wc or word or layout" 2>&1 | tail -1
python tools/wc_overhead.py 4
for cfg in "4 256" "6 256" "8 256"; do set -- $cfg
  timeout 300 python bench.py --workload wordcount --gather zc --slots $1 --lane-bytes $2 --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/wc6_$1_$2.json 2>gpurun_out/wc6.err
  python3 -c "import json;d=json.load(open('gpurun_out/wc6_$1_$2.json'));s=d['stages_ms_per_step'];print('slots=$1 lane=$2', d['value'], d['ms_per_step'], d['config']['n_chunks'], s['ms_h2d'], s['ms_addrgen'], s['ms_gather'], s['ms_compute'], s['ms_device'], d['link']['frac'], d['e2e']['value'], d['overlap']['overlap_frac'])" || tail -3 gpurun_out/wc6.err
done
B="python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-dbuf --no-profile"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_wc" -s 40 -c 1 \
    -o gpurun_out/${TAG}_prof_wc $B --workload wordcount --gather zc > gpurun_out/${TAG}_f5.log 2>&1; tail -1 gpurun_out/${TAG}_f5.log
