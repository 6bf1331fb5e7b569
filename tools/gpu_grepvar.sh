#!/bin/bash
# grep compute variants inside the pipeline: TMA stream (persistent grid), TMA one tile per warp, plain LDG.
mkdir -p gpurun_out
TAG=${TAG:-r01g}
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "grep" --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${TAG}_grep_tests.log 2>&1
tail -2 gpurun_out/${TAG}_grep_tests.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-dbuf"
for v in tma tilegrid ldg; do
  E=""; [ $v = tilegrid ] && E="BK_GREP_TILEGRID=1"; [ $v = ldg ] && E="BK_GREP_LDG=1"
  for rep in 1 2; do
    env $E timeout 600 $B > gpurun_out/${TAG}_$v$rep.json 2> gpurun_out/${TAG}_$v$rep.err
    python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_$v$rep.json'));s=d['stages_ms_per_step'];print('$v', d['value'], d['ms_per_step'], s['ms_compute'], s['ms_zc'], s['ms_h2d'], s['ms_cpu_gather'], d['config']['chunks_cpu_assembled'])" || tail -3 gpurun_out/${TAG}_$v$rep.err
  done
done
