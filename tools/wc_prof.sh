#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-r01b}
(timeout 300 ./build/cpu_gather_probe 16) > gpurun_out/${TAG}_cpu_gather.txt 2>&1
cat gpurun_out/${TAG}_cpu_gather.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_wc$" -s 20 -c 1 \
    -o gpurun_out/${TAG}_prof_wc python bench.py --workload wordcount --steps 1 --warmup 0 --no-cpu-baseline > gpurun_out/${TAG}_ncu_wc.log 2>&1
tail -2 gpurun_out/${TAG}_ncu_wc.log
