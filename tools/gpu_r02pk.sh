#!/bin/bash
# packer prefetch configurations as template constants, in the grep bench (zero-copy traffic running), one box
mkdir -p gpurun_out
T=${TAG:-r02pk}
run() {  dir=$1; name=$2; shift 2
  (cd $dir && env "$@" timeout 900 python bench.py "${ARGS[@]}" > $GRAFT_REPO_ROOT/gpurun_out/${T}_$name.json 2> $GRAFT_REPO_ROOT/gpurun_out/${T}_$name.err)
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_$name.json').read().splitlines()[-1]);s=d['stages_ms_per_step'];print('$name', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'], s['ms_zc'], s['ms_compute'], s['ms_cpu_gather'])" || tail -2 gpurun_out/${T}_$name.err
}
ARGS=(--steps 10 --warmup 3 --no-cpu-baseline --no-dbuf)
for r in 1 2; do
  run bis_c5e0549 c5e_$r BK_X=0
  for cfg in 1 2 3 4 5 6; do run . cfg${cfg}_$r BK_PACK_CFG=$cfg; done
done
ARGS=(--workload groupby_sparse --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf)
for cfg in 1 2 4; do run . sparse_cfg${cfg} BK_PACK_CFG=$cfg; done
run bis_c5e0549 sparse_c5e BK_X=0
