#!/bin/bash
mkdir -p gpurun_out
T=${TAG:-r02p}
timeout 900 python -m pytest tests/test_gpu_kmer.py tests/test_gpu_api_state.py tests/test_gpu_addr.py -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -4 gpurun_out/${T}_tests.log
timeout 900 python bench.py --workload kmer --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/${T}_bench_kmer.json 2> gpurun_out/${T}_bench_kmer.err
python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_kmer.json').read().splitlines()[-1]);t=d['timed_pass_trace'];print('kmer', d['value'], d['ms_per_step'], d['link']['frac'], t['stages_ms'], t['compute_busy_ms'], t['xfer_busy_ms'])" || tail -5 gpurun_out/${T}_bench_kmer.err
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_kmer" -c 40 --csv --log-file gpurun_out/${T}_kmer_launches.csv python bench.py --workload kmer --gib 1 --steps 1 --warmup 0 --no-cpu-baseline --no-dbuf --no-profile --no-trace > /dev/null 2>&1
echo ncu rc=$?
