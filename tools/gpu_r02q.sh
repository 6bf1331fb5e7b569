#!/bin/bash
mkdir -p gpurun_out
T=${TAG:-r02q}
timeout 600 python -m pytest tests/test_gpu_kmer.py -q --timeout 300 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -2 gpurun_out/${T}_tests.log
for g in auto cpu zc; do
timeout 900 python bench.py --workload kmer --gather $g --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/${T}_bench_kmer_$g.json 2> gpurun_out/${T}_bench_kmer_$g.err
python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_kmer_$g.json').read().splitlines()[-1]);t=d['timed_pass_trace'];print('kmer $g', d['value'], d['ms_per_step'], d['link']['frac'], t['stages_ms'], t['compute_busy_ms'], t['xfer_busy_ms'], t['overlap_ms'])" || tail -5 gpurun_out/${T}_bench_kmer_$g.err
done
