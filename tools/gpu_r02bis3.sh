#!/bin/bash
# grep bisect c235fc2..HEAD, one box, interleaved
mkdir -p gpurun_out
T=${TAG:-r02bis3}
run() {  dir=$1; name=$2; shift 2
  (cd $dir && env "$@" timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-dbuf > $GRAFT_REPO_ROOT/gpurun_out/${T}_$name.json 2> $GRAFT_REPO_ROOT/gpurun_out/${T}_$name.err)
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_$name.json').read().splitlines()[-1]);s=d['stages_ms_per_step'];print('$name', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'], s['ms_zc'], s['ms_compute'], s['ms_cpu_gather'])" || tail -2 gpurun_out/${T}_$name.err
}
for r in 1 2; do
  run bis_c235fc2 c23_$r BK_X=0
  run bis_c5e0549 c5e_$r BK_X=0
  run bis_dda7c46 dda_$r BK_X=0
  run bis_dda7c46 ddaopf_$r BK_PACK_PF=16 BK_PACK_PF2=0 BK_PACK_PFEND=0
  run bis_ae46baf ae4_$r BK_X=0
  run bis_4bc29be 4bc_$r BK_X=0
done
