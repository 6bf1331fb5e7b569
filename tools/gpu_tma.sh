#!/bin/bash
# TMA-staged compute kernels: parity, bench lines, ncu of the new kernels.
mkdir -p gpurun_out
TAG=${TAG:-r01t}
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -3 gpurun_out/${TAG}_gpu_tests.log
for w in grep groupby kmeans; do
  S=5; [ $w != grep ] && S=3
  timeout 900 python bench.py --workload $w --steps $S --warmup 3 > gpurun_out/${TAG}_bench_$w.json 2> gpurun_out/${TAG}_bench_$w.err
  python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_$w.json'));print('$w', d['value'], d['ms_per_step'], d['link']['frac'], d['roofline']['kernel'], round(d['roofline']['frac'],4), d['stages_ms_per_step'], d['clocks']['reasons'])" || tail -5 gpurun_out/${TAG}_bench_$w.err
done
B="python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-dbuf --no-profile"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_grep_count|k_grep_write|k_grep_scan" -s 6 -c 3 \
    -o gpurun_out/${TAG}_prof_grep $B --gib 4 > gpurun_out/${TAG}_f1.log 2>&1; tail -1 gpurun_out/${TAG}_f1.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_groupby" -s 4 -c 1 \
    -o gpurun_out/${TAG}_prof_groupby $B --workload groupby --gib 4 > gpurun_out/${TAG}_f2.log 2>&1; tail -1 gpurun_out/${TAG}_f2.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_kmeans" -s 2 -c 1 \
    -o gpurun_out/${TAG}_prof_kmeans $B --workload kmeans --gib 2 > gpurun_out/${TAG}_f3.log 2>&1; tail -1 gpurun_out/${TAG}_f3.log
