#!/bin/bash
# Quick confirmation on a fresh box: GPU parity suite + the default bench line.
mkdir -p gpurun_out
TAG=${TAG:-r01q}
timeout 900 python -m pytest tests -m gpu -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -2 gpurun_out/${TAG}_gpu_tests.log
timeout 900 python bench.py > gpurun_out/${TAG}_bench_grep.json 2> gpurun_out/${TAG}_bench_grep.err
python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_grep.json'));print('grep', d['value'], d['ms_per_step'], d['link']['frac'], d['roofline']['frac'], d['clocks'])" || tail -5 gpurun_out/${TAG}_bench_grep.err
for w in $EXTRA; do
  timeout 900 python bench.py --workload $w > gpurun_out/${TAG}_bench_$w.json 2> gpurun_out/${TAG}_bench_$w.err
  python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_$w.json'));print('$w', d['value'], d['ms_per_step'], d['link']['frac'], d['roofline']['kernel'], round(d['roofline']['frac'],4))" || tail -5 gpurun_out/${TAG}_bench_$w.err
done
