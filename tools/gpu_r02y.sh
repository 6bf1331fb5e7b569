#!/bin/bash
# grep A/B on one box: round-1 tree vs now (default packer prefetch / round-1 prefetch)
mkdir -p gpurun_out
T=${TAG:-r02y}
old() {
  (cd ab_r01 && timeout 900 python bench.py --steps 10 --warmup 3 > ../gpurun_out/${T}_ab_old$1.json 2> ../gpurun_out/${T}_ab_old$1.err)
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_ab_old$1.json').read().splitlines()[-1]);s=d['stages_ms_per_step'];print('old', d['value'], d['ms_per_step'], s.get('ms_cpu_gather'), s.get('ms_zc'), s.get('ms_h2d'), d['config']['chunks_cpu_assembled'], (d.get('cpu_mt_baseline') or {}).get('value'))" || tail -3 gpurun_out/${T}_ab_old$1.err
}
new() {  name=$1; shift
  env "$@" timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/${T}_$name.json 2> gpurun_out/${T}_$name.err
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_$name.json').read().splitlines()[-1]);s=d['stages_ms_per_step'];print('$name', d['value'], d['ms_per_step'], s.get('ms_cpu_gather'), s.get('ms_zc'), s.get('ms_h2d'), d['config']['chunks_cpu_assembled'], (d.get('cpu_mt_baseline') or {}).get('value'))" || tail -3 gpurun_out/${T}_$name.err
}
old 1
new new_pf_r01 BK_PACK_PF=16 BK_PACK_PF2=0 BK_PACK_PFEND=0
new new_default BK_X=0
new new_pf_near BK_PACK_PF=16 BK_PACK_PF2=0 BK_PACK_PFEND=1
new new_pf_r01b BK_PACK_PF=16 BK_PACK_PF2=0 BK_PACK_PFEND=0
old 2
