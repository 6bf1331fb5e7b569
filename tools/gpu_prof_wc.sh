#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-r01w}
python -m pytest tests -m gpu -x -q 2>&1 | tail -2
B="python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-dbuf --no-profile"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_wc|k_gather_whole|k_lane_first|k_addrgen" -s 40 -c 4 \
    -o gpurun_out/${TAG}_prof_wc $B --workload wordcount --gather zc > gpurun_out/${TAG}_f5.log 2>&1; tail -1 gpurun_out/${TAG}_f5.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_kmer" -s 6 -c 1 \
    -o gpurun_out/${TAG}_prof_kmer $B --workload kmer --gib 1 > gpurun_out/${TAG}_f6.log 2>&1; tail -1 gpurun_out/${TAG}_f6.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_wc.csv \
    $B --workload wordcount --gather zc > gpurun_out/${TAG}_l5.log 2>&1; tail -c 300 gpurun_out/${TAG}_l5.log
