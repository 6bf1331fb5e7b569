#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-r01v}
timeout 1200 python -m pytest tests -m gpu -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -3 gpurun_out/${TAG}_gpu_tests.log
timeout 900 python bench.py --workload kmeans --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_kmeans.json 2> gpurun_out/${TAG}_bench_kmeans.err
python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_kmeans.json'));print('kmeans', d['value'], d['ms_per_step'], d['stages_ms_per_step']['ms_compute'])" || tail -5 gpurun_out/${TAG}_bench_kmeans.err
B="python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-dbuf --no-profile"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_kmeans" -s 2 -c 1 \
    -o gpurun_out/${TAG}_prof_kmeans $B --workload kmeans --gib 2 > gpurun_out/${TAG}_f3.log 2>&1; tail -1 gpurun_out/${TAG}_f3.log
