#!/bin/bash
# two-phase k-mer counting: tests + bench
mkdir -p gpurun_out
T=${TAG:-r02m}
timeout 900 python -m pytest tests/test_gpu_kmer.py tests/test_gpu_api_state.py tests/test_gpu_addr.py -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -6 gpurun_out/${T}_tests.log
timeout 900 python bench.py --workload kmer --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/${T}_bench_kmer.json 2> gpurun_out/${T}_bench_kmer.err
python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_kmer.json').read().splitlines()[-1]);t=d['timed_pass_trace'];print('kmer', d['value'], d['ms_per_step'], d['link']['frac'], t['stages_ms'], t['compute_busy_ms'], t['xfer_busy_ms'])" || tail -5 gpurun_out/${T}_bench_kmer.err
