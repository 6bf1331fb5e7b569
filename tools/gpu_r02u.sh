#!/bin/bash
# k-mer flush with 32-bit shared counts (2 CTAs/SM), one flush by default; placement sweep
mkdir -p gpurun_out
T=${TAG:-r02u}
timeout 900 python -m pytest tests/test_gpu_kmer.py -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
tail -3 gpurun_out/${T}_tests.log
line() {  name=$1; shift
  timeout 1500 python bench.py "$@" > gpurun_out/${T}_bench_$name.json 2> gpurun_out/${T}_bench_$name.err
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_$name.json').read().splitlines()[-1]);r=d['roofline'];t=d.get('timed_pass_trace') or {};print('$name', d['value'], d['ms_per_step'], round(r['frac'],3), d['link']['frac'], d['config']['chunks_cpu_assembled'], d['config']['n_chunks'], t.get('device_span_ms'), (t.get('stages_ms') or {}).get('ms_compute'), t.get('overlap_frac'))" || tail -3 gpurun_out/${T}_bench_$name.err
}
line kmer --workload kmer --steps 3 --warmup 3 --no-cpu-baseline
BK_KMER_SPLIT_EACH=1 line kmer_se --workload kmer --steps 3 --warmup 3 --no-cpu-baseline
BK_KMER_F=8 line kmer_f8 --workload kmer --steps 3 --warmup 3 --no-cpu-baseline
BK_KMER_SPLIT_EACH=1 BK_KMER_F=8 line kmer_se_f8 --workload kmer --steps 3 --warmup 3 --no-cpu-baseline
BK_KMER_SPLIT_EACH=1 BK_KMER_F=4 line kmer_se_f4 --workload kmer --steps 3 --warmup 3 --no-cpu-baseline
for v in 0 1; do
  BK_KMER_SPLIT_EACH=$v timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv \
      --log-file gpurun_out/${T}_launches_kmer_se$v.csv python bench.py --workload kmer --steps 1 --warmup 1 \
      --no-cpu-baseline --no-dbuf --no-profile --no-trace > /dev/null 2>&1
  echo "launches kmer se=$v rc=$?"
  python3 tools/ncu_summary.py launches gpurun_out/${T}_launches_kmer_se$v.csv | head -12
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_kmer_flush" -s 1 -c 1 -o gpurun_out/${T}_kflush \
   python bench.py --workload kmer --gib 1 --steps 1 --warmup 1 --no-cpu-baseline --no-dbuf --no-profile --no-trace > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_kmer_bin" -s 6 -c 1 -o gpurun_out/${T}_kbin \
   python bench.py --workload kmer --gib 1 --steps 1 --warmup 1 --no-cpu-baseline --no-dbuf --no-profile --no-trace > /dev/null 2>&1
echo ncu rc=$?
