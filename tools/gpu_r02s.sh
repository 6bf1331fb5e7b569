#!/bin/bash
# HYBRID fix + k-mer block binning: tests, the affected bench lines, packer prefetch sweep, sanitizers
mkdir -p gpurun_out
T=${TAG:-r02s}
timeout 900 python -m pytest tests/test_gpu_kmer.py tests/test_gpu_api_state.py -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -3 gpurun_out/${T}_tests.log
line() {  name=$1; shift
  timeout 1500 python bench.py "$@" > gpurun_out/${T}_bench_$name.json 2> gpurun_out/${T}_bench_$name.err
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_$name.json').read().splitlines()[-1]);r=d['roofline'];print('$name', d['value'], d['ms_per_step'], round(r['frac'],3), d['link']['frac'], (r.get('hybrid_schedule') or {}).get('frac'), d['config']['chunks_cpu_assembled'], d['config']['n_chunks'])" || tail -3 gpurun_out/${T}_bench_$name.err
}
line grep --steps 10 --warmup 3
line groupby_sparse --workload groupby_sparse --steps 3 --warmup 3
line kmer --workload kmer --steps 3 --warmup 3
line grep_ht2_hybrid --host-threads 2 --gib 4 --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf
line grep_ht2_zc --gather zc --host-threads 2 --gib 4 --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf
line grep_ht8_hybrid --host-threads 8 --gib 4 --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf
line grep_ht8_zc --gather zc --host-threads 8 --gib 4 --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf
line grep_addr --gather addr --gib 2 --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf
bash tools/gpu_r02r.sh
TAG=${T} bash tools/sanitize.sh
