#!/bin/bash
# Round-2 final evidence for the lines the last HYBRID change touches (through gpurun): the GPU
# suite file by file, smoke, the HYBRID bench lines (grep = the default line, sparse group-by,
# k-mers, a rank's share of host threads at P = 8 / 2), the reference arm, launch lists.
mkdir -p gpurun_out
T=${TAG:-r02fin}
for f in tests/test_gpu_*.py; do
  b=$(basename $f .py)
  timeout 1500 python -m pytest $f -v --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_$b.log 2>&1
  echo "$b rc=$? $(grep -cE 'PASSED' gpurun_out/${T}_$b.log) passed $(grep -cE 'FAILED' gpurun_out/${T}_$b.log) failed"
done
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.log 2>&1; tail -1 gpurun_out/${T}_smoke.log
line() {
  name=$1; shift
  timeout 1500 python bench.py "$@" > gpurun_out/${T}_bench_$name.json 2> gpurun_out/${T}_bench_$name.err
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_bench_$name.json').read().splitlines()[-1]);print('$name', d['value'], d['ms_per_step'], round(d['roofline']['frac'],3), d['link']['frac'])" \
    || tail -3 gpurun_out/${T}_bench_$name.err
}
line grep --steps 10 --warmup 3
line groupby_sparse --workload groupby_sparse --steps 3 --warmup 3
line kmer --workload kmer --steps 3 --warmup 3
line grep_ht2_hybrid --host-threads 2 --gib 4 --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf
line grep_ht2_zc --gather zc --host-threads 2 --gib 4 --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf
line grep_ht8_hybrid --host-threads 8 --gib 4 --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf
line grep_ht8_zc --gather zc --host-threads 8 --gib 4 --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf
line grep_default_5steps
timeout 900 python bench.py --impl reference > gpurun_out/${T}_bench_reference.json 2> gpurun_out/${T}_bench_reference.err
tail -c 200 gpurun_out/${T}_bench_reference.json
for w in grep kmer; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
      --log-file gpurun_out/${T}_launches_$w.csv python bench.py --workload $w --steps 2 --warmup 1 \
      --no-cpu-baseline --no-dbuf --no-profile --no-trace --gib $([ $w = grep ] && echo 2 || echo 1) > /dev/null 2>&1
  echo "launches $w rc=$?"
done
