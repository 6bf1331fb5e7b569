#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-r01e}
timeout 900 python -m pytest tests -m gpu -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -4 gpurun_out/${TAG}_gpu_tests.log
for cfg in "cpu 16 4" "cpu 8 4" "cpu 12 4" "cpu 16 6" "hybrid 16 4" "hybrid 16 6" "hybrid 12 6" "hybrid 16 8"; do
  set -- $cfg
  timeout 600 python bench.py --gather $1 --host-threads $2 --slots $3 --no-cpu-baseline --steps 4 --warmup 2 > gpurun_out/${TAG}_b_$1_$2_$3.json 2> gpurun_out/${TAG}_b_$1_$2_$3.err
  python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_b_$1_$2_$3.json'));print('$cfg', d['value'], d['ms_per_step'], d['link']['frac'], d['stages_ms_per_step'], d['config']['chunks_cpu_assembled'])" || tail -3 gpurun_out/${TAG}_b_$1_$2_$3.err
done
