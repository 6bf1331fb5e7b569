#!/bin/bash
# EXPERIMENT: k_wc block-table size (BK_WC_TAB) at C1 and at 1 GiB / 128 MiB window.
mkdir -p gpurun_out
TAG=${TAG:-r01wt}
BK_WC_TAB=128 timeout 300 python -m pytest tests/test_gpu_parity.py -q -k "wordcount" -p no:cacheprovider 2>&1 | tail -1
for t in 512 256 128 512 256 128; do
  BK_WC_TAB=$t timeout 300 python bench.py --workload wordcount --steps 30 --warmup 5 --no-cpu-baseline --no-dbuf > gpurun_out/${TAG}_$t.json 2>/dev/null
  python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_$t.json'));print('C1 $t', d['value'], d['ms_per_step'])"
done
for t in 512 128; do
  BK_WC_TAB=$t timeout 300 python bench.py --workload wordcount --steps 5 --warmup 3 --no-cpu-baseline --no-dbuf --gib 1 --window-mib 128 > gpurun_out/${TAG}_big_$t.json 2>/dev/null
  python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_big_$t.json'));print('1GiB $t', d['value'], d['ms_per_step'])"
done
