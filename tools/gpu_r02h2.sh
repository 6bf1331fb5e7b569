#!/bin/bash
# re-run of the r02g test set (segfault there) on the reverted split; fixed zero-copy shares for grep
mkdir -p gpurun_out
T=${TAG:-r02h2}
timeout 1500 python -X faulthandler -m pytest tests/test_gpu_kmer.py tests/test_gpu_parity.py tests/test_gpu_api_state.py tests/test_gpu_edge.py -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
echo "tests rc=$?"; tail -2 gpurun_out/${T}_tests.log
line() {  name=$1; shift
  timeout 1500 python bench.py "$@" > gpurun_out/${T}_bench_$name.json 2> gpurun_out/${T}_bench_$name.err
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_$name.json').read().splitlines()[-1]);r=d['roofline'];print('$name', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'], d['config']['n_chunks'])" || tail -3 gpurun_out/${T}_bench_$name.err
}
for r in 1 2; do
  line grep_auto$r --steps 10 --warmup 3 --no-cpu-baseline --no-dbuf --no-profile
  for z in 150 200 250; do line grep_zc${z}_$r --steps 10 --warmup 3 --no-cpu-baseline --no-dbuf --no-profile --gather hybrid --zc-share $z; done
done
