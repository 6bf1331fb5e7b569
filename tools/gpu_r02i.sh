#!/bin/bash
# CUPTI trace flag + fresh bench lines (all workloads)
mkdir -p gpurun_out
T=${TAG:-r02i}
timeout 900 python -m pytest tests/test_gpu_api_state.py -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -6 gpurun_out/${T}_tests.log
for W in grep wordcount groupby_sparse; do
timeout 900 python bench.py --workload $W --steps 5 --warmup 3 > gpurun_out/${T}_bench_$W.json 2> gpurun_out/${T}_bench_$W.err
python3 - <<PY || tail -5 gpurun_out/${T}_bench_$W.err
import json
d=json.loads(open('gpurun_out/${T}_bench_$W.json').read().splitlines()[-1])
r=d['roofline']
print('$W', d['value'], d['ms_per_step'], 'frac', round(r['frac'],3), 'trace', d.get('timed_pass_trace'))
print('   host', r.get('host_dram'), 'wire', r.get('pcie_wire'))
PY
done
