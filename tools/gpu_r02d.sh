#!/bin/bash
# round 2: fused word count v3 (loader/consumer CTAs, HBM ring): tests, loader sweep, ncu
mkdir -p gpurun_out
T=${TAG:-r02d}
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_api_state.py -k "wordcount" -x -q --timeout 300 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -8 gpurun_out/${T}_tests.log
for L in 16 32 49 74; do
BK_FUSED_LOADERS=$L timeout 300 python bench.py --workload wordcount --steps 20 --warmup 5 --no-cpu-baseline --no-dbuf > gpurun_out/${T}_bench_wc_L$L.json 2> gpurun_out/${T}_bench_wc_L$L.err
python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_wc_L$L.json').read().splitlines()[-1]);print('L=$L', d['value'], d['ms_per_step'], d['roofline'].get('fused'), d['roofline']['frac'])" || tail -5 gpurun_out/${T}_bench_wc_L$L.err
done
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_wc_fused -c 1 -o gpurun_out/${T}_wc_fused python bench.py --workload wordcount --steps 1 --warmup 3 --no-cpu-baseline --no-dbuf --no-profile > gpurun_out/${T}_ncu.log 2>&1
tail -2 gpurun_out/${T}_ncu.log
