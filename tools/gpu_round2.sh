#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-r01c}
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 --tb=short -p no:cacheprovider --durations=5 > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -25 gpurun_out/${TAG}_gpu_tests.log
for g in zc cpu hybrid; do
  timeout 600 python bench.py --gather $g --no-cpu-baseline --steps 5 --warmup 3 > gpurun_out/${TAG}_bench_grep_$g.json 2> gpurun_out/${TAG}_bench_grep_$g.err
  python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_grep_$g.json'));print('$g', d['value'], d['ms_per_step'], d['link'], d['stages_ms_per_step'], d['config']['chunks_cpu_assembled'], d['roofline']['frac'])" || tail -5 gpurun_out/${TAG}_bench_grep_$g.err
done
timeout 300 python bench.py --workload wordcount --no-cpu-baseline > gpurun_out/${TAG}_bench_wc.json 2> gpurun_out/${TAG}_bench_wc.err
python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_wc.json'));print('wc', d['value'], d['ms_per_step'], d['stages_ms_per_step'])" || tail -5 gpurun_out/${TAG}_bench_wc.err
