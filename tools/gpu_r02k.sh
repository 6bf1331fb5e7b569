#!/bin/bash
# fused word count fed by the copy engine (stream-ordered flags): tests + K sweep vs zero-copy loaders
mkdir -p gpurun_out
T=${TAG:-r02k}
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_api_state.py "tests/test_gpu_ranks_parity.py::test_wordcount_two_ranks" -k "wordcount" -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -6 gpurun_out/${T}_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
for cfg in "dma 2" "dma 3" "dma 4" "zc 3"; do set -- $cfg
BK_FUSED_FEED=$1 BK_FUSED_BATCHES=$2 timeout 300 python bench.py --workload wordcount --steps 20 --warmup 5 --no-cpu-baseline --no-dbuf > gpurun_out/${T}_bench_wc_$1$2.json 2> gpurun_out/${T}_bench_wc_$1$2.err
python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_wc_$1$2.json').read().splitlines()[-1]);f=d['roofline'].get('fused');t=d.get('timed_pass_trace') or {};print('$1 K=$2', d['value'], d['ms_per_step'], 'link', d['link']['frac'], 'kern', round(d['roofline']['frac'],3), f['consumer_wait_frac'], f['consumer_compute_frac'], t.get('stages_ms'), t.get('span_vs_ms_per_step'))" || tail -5 gpurun_out/${T}_bench_wc_$1$2.err
done
