#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-r01k}
for lb in 0 96 192 0; do
  timeout 600 python bench.py --workload kmer --steps 3 --warmup 2 --no-cpu-baseline --lane-bytes $lb > gpurun_out/${TAG}_kmer_$lb.json 2> gpurun_out/${TAG}_kmer_$lb.err
  python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_kmer_$lb.json'));s=d['stages_ms_per_step'];print('$lb', d['value'], d['ms_per_step'], s['ms_compute'], d['overlap']['compute_busy_ms'], d['config']['lanes_per_chunk'])" || tail -3 gpurun_out/${TAG}_kmer_$lb.err
done
timeout 600 ncu --set full --clock-control none -k regex:"k_kmer$" -s 6 -c 1 -o gpurun_out/${TAG}_prof_kmer96 python bench.py --workload kmer --gib 1 --steps 1 --warmup 0 --no-cpu-baseline --no-profile --lane-bytes 96 > gpurun_out/${TAG}_f.log 2>&1; tail -1 gpurun_out/${TAG}_f.log
