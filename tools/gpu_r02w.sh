#!/bin/bash
# word count: warp-aggregated compaction stored straight into the caller's arrays
mkdir -p gpurun_out
T=${TAG:-r02w}
timeout 1200 python -m pytest tests/test_gpu_parity.py -k "wordcount or dbuf" tests/test_gpu_api_state.py tests/test_gpu_ranks_parity.py tests/test_gpu_merge.py tests/test_gpu_edge.py -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -3 gpurun_out/${T}_tests.log
line() {  name=$1; shift
  timeout 1500 python bench.py "$@" > gpurun_out/${T}_bench_$name.json 2> gpurun_out/${T}_bench_$name.err
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_$name.json').read().splitlines()[-1]);t=d.get('timed_pass_trace') or {};print('$name', d['value'], d['ms_per_step'], d['link']['frac'], t.get('device_span_ms'), d['e2e']['value'])" || tail -3 gpurun_out/${T}_bench_$name.err
}
line wordcount --workload wordcount --steps 20 --warmup 5
line wordcount2 --workload wordcount --steps 50 --warmup 10
timeout 600 python tools/wc_overhead.py
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
      --log-file gpurun_out/${T}_launches_wordcount.csv python bench.py --workload wordcount --steps 2 --warmup 1 \
      --no-cpu-baseline --no-dbuf --no-profile --no-trace > /dev/null 2>&1
python3 tools/ncu_summary.py launches gpurun_out/${T}_launches_wordcount.csv | head -8
