#!/bin/bash
# word count: block-staged compaction into the caller's arrays; grep A/B: round-1 tree vs now, same box
mkdir -p gpurun_out
T=${TAG:-r02x}
timeout 1200 python -m pytest tests/test_gpu_parity.py -k "wordcount or dbuf" tests/test_gpu_ranks_parity.py tests/test_gpu_merge.py -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -2 gpurun_out/${T}_tests.log
line() {  name=$1; shift
  timeout 1500 python bench.py "$@" > gpurun_out/${T}_bench_$name.json 2> gpurun_out/${T}_bench_$name.err
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_$name.json').read().splitlines()[-1]);t=d.get('timed_pass_trace') or {};print('$name', d['value'], d['ms_per_step'], d['link']['frac'], t.get('device_span_ms'), d['e2e']['value'], (d.get('cpu_mt_baseline') or {}).get('value'))" || tail -3 gpurun_out/${T}_bench_$name.err
}
line wordcount --workload wordcount --steps 20 --warmup 5
timeout 600 python tools/wc_overhead.py
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
      --log-file gpurun_out/${T}_launches_wordcount.csv python bench.py --workload wordcount --steps 2 --warmup 1 \
      --no-cpu-baseline --no-dbuf --no-profile --no-trace > /dev/null 2>&1
python3 tools/ncu_summary.py launches gpurun_out/${T}_launches_wordcount.csv | head -8
for rep in 1 2; do
  (cd ab_r01 && timeout 900 python bench.py --steps 10 --warmup 3 > ../gpurun_out/${T}_ab_old$rep.json 2> ../gpurun_out/${T}_ab_old$rep.err)
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_ab_old$rep.json').read().splitlines()[-1]);print('old', d['value'], d['ms_per_step'], d['stages_ms_per_step'].get('ms_cpu_gather'), d['config']['chunks_cpu_assembled'], (d.get('cpu_mt_baseline') or {}).get('value'))" || tail -3 gpurun_out/${T}_ab_old$rep.err
  line grep_new$rep --steps 10 --warmup 3
done
