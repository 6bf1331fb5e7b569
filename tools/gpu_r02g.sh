#!/bin/bash
# HYBRID split from the link/host balance model; new capacity tests
mkdir -p gpurun_out
T=${TAG:-r02g}
timeout 1500 python -m pytest tests/test_gpu_kmer.py tests/test_gpu_parity.py tests/test_gpu_api_state.py tests/test_gpu_edge.py -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -2 gpurun_out/${T}_tests.log
line() {  name=$1; shift
  timeout 1500 python bench.py "$@" > gpurun_out/${T}_bench_$name.json 2> gpurun_out/${T}_bench_$name.err
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_$name.json').read().splitlines()[-1]);r=d['roofline'];h=r.get('hybrid_schedule') or {};print('$name', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'], d['config']['n_chunks'], h.get('frac'), h.get('x_zc_opt'), h.get('x_zc_run'))" || tail -3 gpurun_out/${T}_bench_$name.err
}
(cd ab_r01 && timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-dbuf > ../gpurun_out/${T}_r01tree.json 2>/dev/null) && python3 -c "import json;d=json.loads(open('gpurun_out/${T}_r01tree.json').read().splitlines()[-1]);print('r01tree', d['value'])"
line grep --steps 10 --warmup 3 --no-cpu-baseline --no-dbuf
line grep2 --steps 10 --warmup 3 --no-cpu-baseline --no-dbuf
line groupby_sparse --workload groupby_sparse --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf
line kmer --workload kmer --steps 3 --warmup 3 --no-cpu-baseline
line grep_ht2_hybrid --host-threads 2 --gib 4 --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf
line grep_ht8_hybrid --host-threads 8 --gib 4 --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf
