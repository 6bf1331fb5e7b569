#!/bin/bash
# ncu evidence for profiles/: launch lists (serialised, cold) + one --set full capture per top kernel.
mkdir -p gpurun_out
TAG=${TAG:-r01n}
B="python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-dbuf"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_grep.csv \
    $B --zc-share 333 > gpurun_out/${TAG}_l1.log 2>&1; tail -c 300 gpurun_out/${TAG}_l1.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_groupby.csv \
    $B --workload groupby --gib 4 > gpurun_out/${TAG}_l2.log 2>&1; tail -1 gpurun_out/${TAG}_l2.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_gather_field|k_grep_count|k_grep_write" -s 2 -c 3 \
    -o gpurun_out/${TAG}_prof_grep $B --zc-share 1000 --gib 4 > gpurun_out/${TAG}_f1.log 2>&1; tail -1 gpurun_out/${TAG}_f1.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_gather_whole|k_groupby" -s 4 -c 2 \
    -o gpurun_out/${TAG}_prof_groupby $B --workload groupby --gib 4 > gpurun_out/${TAG}_f2.log 2>&1; tail -1 gpurun_out/${TAG}_f2.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_kmeans" -s 2 -c 1 \
    -o gpurun_out/${TAG}_prof_kmeans $B --workload kmeans --gib 2 > gpurun_out/${TAG}_f3.log 2>&1; tail -1 gpurun_out/${TAG}_f3.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_part" -s 8 -c 4 \
    -o gpurun_out/${TAG}_prof_partition $B --workload partition --gib 2 > gpurun_out/${TAG}_f4.log 2>&1; tail -1 gpurun_out/${TAG}_f4.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_wc$" -s 20 -c 1 \
    -o gpurun_out/${TAG}_prof_wc $B --workload wordcount > gpurun_out/${TAG}_f5.log 2>&1; tail -1 gpurun_out/${TAG}_f5.log
