#!/bin/bash
mkdir -p gpurun_out
./build/hgb 16 16 pack | tail -2; ./build/hgb 16 16 | tail -1
python -m pytest tests -m gpu -x -q -k "cpu or hybrid or layout or grep or groupby or kmer" 2>&1 | tail -2
for g in hybrid cpu; do
  timeout 600 python bench.py --gather $g --steps 4 --warmup 3 --no-cpu-baseline --no-dbuf > gpurun_out/pack_$g.json 2>gpurun_out/pack.err
  python3 -c "import json;d=json.load(open('gpurun_out/pack_$g.json'));print('grep $g', d['value'], d['ms_per_step'], d['link']['frac'], d['config']['chunks_cpu_assembled'], d['stages_ms_per_step'], d['overlap']['overlap_frac'])" || tail -3 gpurun_out/pack.err
done
for w in groupby_sparse kmer; do
  timeout 600 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf > gpurun_out/pack_$w.json 2>gpurun_out/pack.err
  python3 -c "import json;d=json.load(open('gpurun_out/pack_$w.json'));print('$w', d['value'], d['ms_per_step'], d['link']['frac'], d['config']['chunks_cpu_assembled'], d['config']['n_chunks'])" || tail -3 gpurun_out/pack.err
done
