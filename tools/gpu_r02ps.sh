#!/bin/bash
mkdir -p gpurun_out
T=r02ps
for r in 1 2; do for sl in 0 6 8 12; do
  timeout 900 python bench.py --workload partition --steps 3 --warmup 3 --no-cpu-baseline --no-profile --no-trace --slots $sl > gpurun_out/${T}_s${sl}_$r.json 2> gpurun_out/${T}_s${sl}_$r.err
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_s${sl}_$r.json').read().splitlines()[-1]);f=d.get('link_full_duplex') or {};print('slots $sl', d['value'], d['ms_per_step'], d['config']['n_chunks'], d['config']['n_slots'], f.get('frac'), f.get('peak_each_way_gbs'))" || tail -2 gpurun_out/${T}_s${sl}_$r.err
done; done
