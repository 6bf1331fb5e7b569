#!/bin/bash
# Fig. 5-style ablation on B200: the same workload through each variant.
mkdir -p gpurun_out
TAG=${TAG:-r01o}
for W in ${WS:-grep}; do
  S=3; [ $W = wordcount ] && S=20
  for v in "sbuf auto" "dbuf auto" "ours dense" "ours zc" "ours cpu" "ours hybrid"; do
    set -- $v
    timeout 600 python bench.py --workload $W --impl $1 --gather $2 --steps $S --warmup 3 --no-cpu-baseline --no-dbuf > gpurun_out/${TAG}_${W}_$1_$2.json 2> gpurun_out/${TAG}_${W}_$1_$2.err
    python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_${W}_$1_$2.json'));print('| $W | $1 | $2 |', d['value'], '|', d['ms_per_step'], '|', d['link']['frac'], '|', d['link']['bytes_per_step_per_gpu'], '|')" || tail -1 gpurun_out/${TAG}_${W}_$1_$2.err
  done
done
