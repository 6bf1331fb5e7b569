#!/bin/bash
# grep A/B on one box, interleaved: round-1 tree / now / now with the round-1 HYBRID depth and prefetch
mkdir -p gpurun_out
T=${TAG:-r02z2}
old() {
  (cd ab_r01 && timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-dbuf > ../gpurun_out/${T}_old$1.json 2> ../gpurun_out/${T}_old$1.err)
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_old$1.json').read().splitlines()[-1]);print('old$1', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'])" || tail -3 gpurun_out/${T}_old$1.err
}
new() {  name=$1; shift
  env "$@" timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-dbuf --no-trace > gpurun_out/${T}_$name.json 2> gpurun_out/${T}_$name.err
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_$name.json').read().splitlines()[-1]);print('$name', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'], d['step_ms'])" || tail -3 gpurun_out/${T}_$name.err
}
for r in 1 2 3; do
  old $r
  new new$r BK_X=0
  new fixed$r BK_HYBRID_DEPTH=1 BK_PACK_PF=16 BK_PACK_PF2=0 BK_PACK_PFEND=0
done
