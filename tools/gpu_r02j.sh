#!/bin/bash
# bench lines: grep (composite roofline), k-means K=64/256, k-mers, partition, group-by 16/32 GiB
mkdir -p gpurun_out
T=${TAG:-r02j}
run() { name=$1; shift; timeout 1200 python bench.py "$@" > gpurun_out/${T}_bench_$name.json 2> gpurun_out/${T}_bench_$name.err
python3 - <<PY || tail -5 gpurun_out/${T}_bench_$name.err
import json
d=json.loads(open('gpurun_out/${T}_bench_$name.json').read().splitlines()[-1])
r=d['roofline']; t=d.get('timed_pass_trace') or {}
print('$name', d['value'], d['ms_per_step'], 'roof', r['kernel'][:40], round(r['frac'],3), 'link', d['link']['frac'], 'trace_span', t.get('span_vs_ms_per_step'), 'ovl', t.get('overlap_frac'), 'stages', t.get('stages_ms'))
for k in ('hybrid_schedule','host_dram','pcie_wire'):
    if k in r: print('   ',k, {a:(round(b,4) if isinstance(b,float) else b) for a,b in r[k].items() if a not in ('note','peak_source')})
PY
}
run grep --steps 5 --warmup 3
run kmeans --workload kmeans --steps 3 --warmup 3
run kmeans256 --workload kmeans --K 256 --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf
run kmer --workload kmer --steps 3 --warmup 3
run partition --workload partition --steps 3 --warmup 3
run groupby --workload groupby --steps 3 --warmup 3
run groupby32 --workload groupby --gib 32 --steps 3 --warmup 3 --no-cpu-baseline
