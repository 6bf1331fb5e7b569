#!/bin/bash
# GPU check after the per-slot staging-stream change: full GPU suite, WC breakdown + sweep, grep/kmer benches.
mkdir -p gpurun_out
python -m pytest tests -m gpu -x -q 2>&1 | tail -4
python tools/wc_overhead.py 4; python tools/wc_overhead.py 3
for sub in 4 8; do for cfg in "4 256" "3 256" "2 256" "4 128"; do set -- $cfg
  BK_WC_SUB=$sub timeout 300 python bench.py --workload wordcount --gather zc --slots $1 --lane-bytes $2 --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/wc3_${sub}_$1_$2.json 2>gpurun_out/wc3.err
  python3 -c "import json;d=json.load(open('gpurun_out/wc3_${sub}_$1_$2.json'));s=d['stages_ms_per_step'];print('sub=$sub slots=$1 lane=$2', d['value'], d['ms_per_step'], d['config']['n_chunks'], s['ms_gather'], s['ms_compute'], s['ms_device'], d['link']['frac'], d['e2e']['value'])" || tail -3 gpurun_out/wc3.err
done; done
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/grep_new.json 2>gpurun_out/grep_new.err; tail -c 600 gpurun_out/grep_new.json
timeout 600 python bench.py --workload kmer --steps 3 --warmup 2 --no-cpu-baseline > gpurun_out/kmer_new.json 2>gpurun_out/kmer_new.err; python3 -c "import json;d=json.load(open('gpurun_out/kmer_new.json'));print('kmer', d['value'], d['ms_per_step'], d['stages_ms_per_step'])"
