#!/bin/bash
# full GPU suite + k-means kernel (warp aggregation) ncu at K=64/256
mkdir -p gpurun_out
T=${TAG:-r02l}
timeout 2400 python -m pytest tests -m gpu -q --timeout 900 --tb=short -p no:cacheprovider > gpurun_out/${T}_gpu_tests.log 2>&1
tail -15 gpurun_out/${T}_gpu_tests.log
for K in 64 256; do
timeout 600 ncu --set full --clock-control none -k regex:k_kmeans -s 20 -c 1 -o gpurun_out/${T}_kmeans_K$K python bench.py --workload kmeans --K $K --gib 2 --steps 1 --warmup 3 --no-cpu-baseline --no-dbuf --no-profile --no-trace > gpurun_out/${T}_ncu_K$K.log 2>&1
tail -1 gpurun_out/${T}_ncu_K$K.log
timeout 600 python bench.py --workload kmeans --K $K --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf > gpurun_out/${T}_bench_kmeans_K$K.json 2> gpurun_out/${T}_bench_kmeans_K$K.err
python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_kmeans_K$K.json').read().splitlines()[-1]);t=d['timed_pass_trace'];print('K=$K', d['value'], d['ms_per_step'], t['stages_ms'], t['compute_busy_ms'], d['config']['n_chunks'])" || tail -3 gpurun_out/${T}_bench_kmeans_K$K.err
done
