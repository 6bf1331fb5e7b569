#!/bin/bash
# fused word count v4 (word-parallel consumers) + address mode fixes
mkdir -p gpurun_out
T=${TAG:-r02g}
timeout 900 python -m pytest tests/test_gpu_addr.py tests/test_gpu_parity.py -k "addr or wordcount or api_errors" -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -8 gpurun_out/${T}_tests.log
for L in 12 24 37; do
BK_FUSED_LOADERS=$L timeout 300 python bench.py --workload wordcount --steps 20 --warmup 5 --no-cpu-baseline --no-dbuf > gpurun_out/${T}_bench_wc_L$L.json 2> gpurun_out/${T}_bench_wc_L$L.err
python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_wc_L$L.json').read().splitlines()[-1]);print('L=$L', d['value'], d['ms_per_step'], d['roofline'].get('fused'), d['roofline']['frac'])" || tail -5 gpurun_out/${T}_bench_wc_L$L.err
done
