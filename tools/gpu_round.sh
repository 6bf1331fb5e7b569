#!/bin/bash
# One GPU session: tests, bench lines, ncu launch list + full capture of the top kernels.
set -x
mkdir -p gpurun_out
TAG=${TAG:-r01}
timeout 900 python -m pytest tests -m gpu -q --timeout 600 --tb=short -p no:cacheprovider --durations=8 > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -15 gpurun_out/${TAG}_gpu_tests.log
timeout 600 python bench.py > gpurun_out/${TAG}_bench_grep.json 2> gpurun_out/${TAG}_bench_grep.err
tail -c 3000 gpurun_out/${TAG}_bench_grep.json; tail -5 gpurun_out/${TAG}_bench_grep.err
timeout 300 python bench.py --workload wordcount > gpurun_out/${TAG}_bench_wc.json 2> gpurun_out/${TAG}_bench_wc.err
tail -c 2000 gpurun_out/${TAG}_bench_wc.json; tail -5 gpurun_out/${TAG}_bench_wc.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_grep.csv \
    python bench.py --steps 1 --warmup 0 --no-cpu-baseline > gpurun_out/${TAG}_ncu_list.log 2>&1
tail -3 gpurun_out/${TAG}_ncu_list.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_gather|k_grep_count|k_grep_write" -s 6 -c 3 \
    -o gpurun_out/${TAG}_prof_grep python bench.py --steps 1 --warmup 0 --gib 4 --no-cpu-baseline > gpurun_out/${TAG}_ncu_full.log 2>&1
tail -3 gpurun_out/${TAG}_ncu_full.log
ls -la gpurun_out
