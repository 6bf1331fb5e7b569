#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-r01x}
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 --tb=short -p no:cacheprovider > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -15 gpurun_out/${TAG}_gpu_tests.log
timeout 900 python bench.py --workload kmeans --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_kmeans.json 2> gpurun_out/${TAG}_bench_kmeans.err
python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_kmeans.json'));print('kmeans', d['value'], d['ms_per_step'], d.get('baseline_dbuf'))" || tail -5 gpurun_out/${TAG}_bench_kmeans.err
