#!/bin/bash
# grep bisect across round-2 commits, one box, interleaved (10 timed steps each)
mkdir -p gpurun_out
T=${TAG:-r02bis}
run() {  dir=$1; name=$2
  (cd $dir && timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-dbuf > $GRAFT_REPO_ROOT/gpurun_out/${T}_$name.json 2> $GRAFT_REPO_ROOT/gpurun_out/${T}_$name.err)
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_$name.json').read().splitlines()[-1]);print('$name', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'])" || tail -2 gpurun_out/${T}_$name.err
}
for r in 1 2; do
  run ab_r01 old$r
  run bis_990faf0 b990$r
  run bis_fee4620 bfee$r
  run bis_dbc49af bdbc$r
  run bis_dab90b5 bdab$r
  run bis_c235fc2 bc23$r
  run . new$r
done
