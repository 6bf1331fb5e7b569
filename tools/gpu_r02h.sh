#!/bin/bash
# fused word count: graph replay, pinned results, loader/unit sweep; Table II measured
mkdir -p gpurun_out
T=${TAG:-r02h}
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_api_state.py -k "wordcount" -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -4 gpurun_out/${T}_tests.log
for U in 16384 32768; do for L in 24 37 49; do
BK_FUSED_UNIT=$U BK_FUSED_LOADERS=$L timeout 300 python bench.py --workload wordcount --steps 20 --warmup 5 --no-cpu-baseline --no-dbuf > gpurun_out/${T}_bench_wc_U${U}_L$L.json 2> gpurun_out/${T}_bench_wc_U${U}_L$L.err
python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_wc_U${U}_L$L.json').read().splitlines()[-1]);f=d['roofline'].get('fused');print('U=$U L=$L', d['value'], d['ms_per_step'], d['roofline']['frac'], f['consumer_wait_frac'], f['consumer_compute_frac'], f['loader_wait_frac'])" || tail -5 gpurun_out/${T}_bench_wc_U${U}_L$L.err
done; done
timeout 900 python tools/table2_measured.py > gpurun_out/${T}_table2.jsonl 2> gpurun_out/${T}_table2.err
cat gpurun_out/${T}_table2.jsonl | cut -c1-400; tail -3 gpurun_out/${T}_table2.err
