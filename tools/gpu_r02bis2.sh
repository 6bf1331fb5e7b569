#!/bin/bash
# grep: which part of the HYBRID change / prefetch costs what, one box, interleaved
mkdir -p gpurun_out
T=${TAG:-r02bis2}
run() {  dir=$1; name=$2; shift 2
  (cd $dir && env "$@" timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-dbuf > $GRAFT_REPO_ROOT/gpurun_out/${T}_$name.json 2> $GRAFT_REPO_ROOT/gpurun_out/${T}_$name.err)
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_$name.json').read().splitlines()[-1]);print('$name', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'])" || tail -2 gpurun_out/${T}_$name.err
}
for r in 1 2; do
  run bis_c235fc2 c23_$r BK_X=0
  run . new_$r BK_X=0
  run . waits_$r BK_HYBRID_TCPU_WAITS=1
  run . waits_oldpf_$r BK_HYBRID_TCPU_WAITS=1 BK_PACK_PF=16 BK_PACK_PF2=0 BK_PACK_PFEND=0
  run . oldpf_$r BK_PACK_PF=16 BK_PACK_PF2=0 BK_PACK_PFEND=0
  run . d2_$r BK_HYBRID_DEPTH=2
done
