#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-r01l}
timeout 900 python -m pytest tests -m gpu -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -3 gpurun_out/${TAG}_gpu_tests.log
timeout 600 python bench.py > gpurun_out/${TAG}_bench_grep.json 2> gpurun_out/${TAG}_bench_grep.err
python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_grep.json'));print('grep', d['value'], d['ms_per_step'], d['link']['frac'], d['baseline_dbuf']['bigkernel_speedup'], d['roofline']['frac'])" || tail -5 gpurun_out/${TAG}_bench_grep.err
timeout 300 python bench.py --workload wordcount > gpurun_out/${TAG}_bench_wordcount.json 2> gpurun_out/${TAG}_bench_wordcount.err
python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_wordcount.json'));print('wc', d['value'], d['ms_per_step'], d['config']['gather_mode'])" || tail -5 gpurun_out/${TAG}_bench_wordcount.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_grep.csv \
    python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-dbuf > gpurun_out/${TAG}_ncu_list.log 2>&1
tail -1 gpurun_out/${TAG}_ncu_list.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_gather|k_grep_count|k_addrgen" -s 3 -c 3 \
    -o gpurun_out/${TAG}_prof_grep python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-dbuf --gib 4 > gpurun_out/${TAG}_ncu_full.log 2>&1
tail -1 gpurun_out/${TAG}_ncu_full.log
