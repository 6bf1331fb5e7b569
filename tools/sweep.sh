#!/bin/bash
# usage: TAG=x bash tools/sweep.sh "gather threads slots [extra args]" ...
mkdir -p gpurun_out
TAG=${TAG:-sweep}
for cfg in "$@"; do
  set -- $cfg
  g=$1; th=$2; sl=$3; shift 3
  name=${TAG}_b_${g}_${th}_${sl}
  timeout 600 python bench.py --gather $g --host-threads $th --slots $sl --no-cpu-baseline --steps 4 --warmup 2 "$@" > gpurun_out/$name.json 2> gpurun_out/$name.err
  python3 -c "import json;d=json.load(open('gpurun_out/$name.json'));print('$cfg', d['value'], d['ms_per_step'], d['link']['frac'], d['stages_ms_per_step'], d['config']['chunks_cpu_assembled'])" || tail -3 gpurun_out/$name.err
done
