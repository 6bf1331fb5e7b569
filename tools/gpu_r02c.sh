#!/bin/bash
# round 2: fused word count v2 (even byte split, per-unit block-table flush): tests, bench, ncu
mkdir -p gpurun_out
T=${TAG:-r02c}
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_api_state.py "tests/test_gpu_ranks_parity.py::test_wordcount_two_ranks" -k "wordcount" -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -8 gpurun_out/${T}_tests.log
timeout 600 python bench.py --workload wordcount --steps 20 --warmup 5 --no-cpu-baseline --no-dbuf > gpurun_out/${T}_bench_wc.json 2> gpurun_out/${T}_bench_wc.err
python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_wc.json').read().splitlines()[-1]);print('fused', d['value'], d['ms_per_step'], d['stages_ms_per_step']['ms_zc'], d['overlap'])" || tail -5 gpurun_out/${T}_bench_wc.err
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_wc_fused -c 1 -o gpurun_out/${T}_wc_fused python bench.py --workload wordcount --steps 1 --warmup 3 --no-cpu-baseline --no-dbuf --no-profile > gpurun_out/${T}_ncu.log 2>&1
tail -3 gpurun_out/${T}_ncu.log
