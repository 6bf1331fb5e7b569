#!/bin/bash
# round 2: fused word count + re-run of the failing tests, then the C1 bench line
mkdir -p gpurun_out
T=${TAG:-r02b}
timeout 900 python -m pytest tests/test_gpu_api_state.py tests/test_gpu_edge.py "tests/test_gpu_ranks_parity.py::test_wordcount_two_ranks" tests/test_gpu_parity.py -k "wordcount or api_state or edge or partition" -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -15 gpurun_out/${T}_tests.log
timeout 600 python bench.py --workload wordcount --steps 20 --warmup 5 > gpurun_out/${T}_bench_wc.json 2> gpurun_out/${T}_bench_wc.err
tail -c 1500 gpurun_out/${T}_bench_wc.json; tail -3 gpurun_out/${T}_bench_wc.err
timeout 600 python bench.py --workload wordcount --gather zc --steps 20 --warmup 5 --no-cpu-baseline --no-dbuf > gpurun_out/${T}_bench_wc_zc.json 2> gpurun_out/${T}_bench_wc_zc.err
python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_wc_zc.json').read().splitlines()[-1]);print('zc', d['value'], d['ms_per_step'])"
