#!/bin/bash
# Round evidence: GPU tests, every bench line, ncu launch lists and one --set full capture per top kernel.
mkdir -p gpurun_out
TAG=${TAG:-r01f}
{ lscpu; free -g; nproc; } > gpurun_out/${TAG}_host.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -2 gpurun_out/${TAG}_gpu_tests.log
timeout 900 python bench.py > gpurun_out/${TAG}_bench_grep.json 2> gpurun_out/${TAG}_bench_grep.err
python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_grep.json'));print('grep', d['value'], d['ms_per_step'], d['link']['frac'], d['roofline']['frac'], d['clocks'])" || tail -5 gpurun_out/${TAG}_bench_grep.err
for w in wordcount groupby groupby_sparse kmeans partition kmer; do
  S=3; [ $w = wordcount ] && S=50
  timeout 900 python bench.py --workload $w --steps $S --warmup 3 > gpurun_out/${TAG}_bench_$w.json 2> gpurun_out/${TAG}_bench_$w.err
  python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_$w.json'));print('$w', d['value'], d['ms_per_step'], d['link']['frac'], d['roofline']['kernel'], round(d['roofline']['frac'],4), d.get('cpu_baseline',{}).get('value'), d['clocks']['samples'], d['clocks']['reasons'])" || tail -5 gpurun_out/${TAG}_bench_$w.err
done
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/${TAG}_bench_reference.json 2> gpurun_out/${TAG}_bench_reference.err; tail -c 300 gpurun_out/${TAG}_bench_reference.json
B="python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-dbuf"
# under ncu kernels serialise, so the adaptive HYBRID split would go all zero-copy: pin the bench's split (9 of 33)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_grep.csv $B --zc-share 273 > gpurun_out/${TAG}_l1.log 2>&1; tail -1 gpurun_out/${TAG}_l1.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_groupby.csv $B --workload groupby --gib 4 > gpurun_out/${TAG}_l2.log 2>&1; tail -1 gpurun_out/${TAG}_l2.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_wordcount.csv $B --workload wordcount > gpurun_out/${TAG}_l3.log 2>&1; tail -1 gpurun_out/${TAG}_l3.log
B="$B --no-profile"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_gather_field|k_grep_count|k_grep_write" -s 2 -c 3 \
    -o gpurun_out/${TAG}_prof_grep $B --zc-share 1000 --gib 4 > gpurun_out/${TAG}_f1.log 2>&1; tail -1 gpurun_out/${TAG}_f1.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_gather_whole|k_groupby" -s 4 -c 2 \
    -o gpurun_out/${TAG}_prof_groupby $B --workload groupby --gib 4 > gpurun_out/${TAG}_f2.log 2>&1; tail -1 gpurun_out/${TAG}_f2.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_kmeans" -s 2 -c 1 \
    -o gpurun_out/${TAG}_prof_kmeans $B --workload kmeans --gib 2 > gpurun_out/${TAG}_f3.log 2>&1; tail -1 gpurun_out/${TAG}_f3.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_part" -s 8 -c 4 \
    -o gpurun_out/${TAG}_prof_partition $B --workload partition --gib 2 > gpurun_out/${TAG}_f4.log 2>&1; tail -1 gpurun_out/${TAG}_f4.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_wc|k_gather_whole|k_lane_first|k_addrgen" -s 40 -c 4 \
    -o gpurun_out/${TAG}_prof_wc $B --workload wordcount --gather zc > gpurun_out/${TAG}_f5.log 2>&1; tail -1 gpurun_out/${TAG}_f5.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_kmer" -s 6 -c 1 \
    -o gpurun_out/${TAG}_prof_kmer $B --workload kmer --gib 1 > gpurun_out/${TAG}_f6.log 2>&1; tail -1 gpurun_out/${TAG}_f6.log
