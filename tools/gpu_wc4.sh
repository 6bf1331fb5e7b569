#!/bin/bash
mkdir -p gpurun_out
BK_WC_SUB=16 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "wc or word" 2>&1 | tail -2
for sub in 8 16; do for cfg in "4 256" "6 256" "8 256" "8 512" "6 512"; do set -- $cfg
  BK_WC_SUB=$sub timeout 300 python bench.py --workload wordcount --gather zc --slots $1 --lane-bytes $2 --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/wc4_${sub}_$1_$2.json 2>gpurun_out/wc4.err
  python3 -c "import json;d=json.load(open('gpurun_out/wc4_${sub}_$1_$2.json'));s=d['stages_ms_per_step'];print('sub=$sub slots=$1 lane=$2', d['value'], d['ms_per_step'], d['config']['n_chunks'], s['ms_h2d'], s['ms_addrgen'], s['ms_gather'], s['ms_compute'], s['ms_device'], d['link']['frac'], d['e2e']['value'])" || tail -3 gpurun_out/wc4.err
done; done
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/grep_new2.json 2>gpurun_out/grep_new2.err; python3 -c "import json;d=json.load(open('gpurun_out/grep_new2.json'));print('grep', d['value'], d['ms_per_step'], d['overlap'])"
