#!/bin/bash
# HYBRID: zero-copy gathers on their own streams (concurrent with the CPU chunks' DMAs) x ZC depth.
mkdir -p gpurun_out
TAG=${TAG:-r01h}
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-dbuf"
for cfg in "base:1:0:4" "own:1:1:4" "own:2:1:4" "own:3:1:4" "own:2:1:6" "own:4:1:8" "base:1:0:4"; do
  IFS=: read name depth own slots <<< "$cfg"
  E="BK_ZC_DEPTH=$depth"; [ $own = 1 ] && E="$E BK_HYBRID_OWNSTREAM=1"
  env $E timeout 600 $B --slots $slots > gpurun_out/${TAG}_${name}_${depth}_${slots}.json 2> gpurun_out/${TAG}_${name}_${depth}_${slots}.err
  python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_${name}_${depth}_${slots}.json'));s=d['stages_ms_per_step'];print('$cfg', d['value'], d['ms_per_step'], 'zc', s['ms_zc'], s['n_zc'], 'h2d', s['ms_h2d'], 'cpu', s['ms_cpu_gather'], d['config']['chunks_cpu_assembled'], d['link']['frac'])" || tail -3 gpurun_out/${TAG}_${name}_${depth}_${slots}.err
done
