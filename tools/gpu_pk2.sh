#!/bin/bash
for cfg in "0 32 16384" "0 8 16384" "0 16 8192" "0 16 4096"; do set -- $cfg
  echo "nt=$1 pf=$2 grab=$3"; BK_PK_NT=$1 BK_PK_PF=$2 BK_PK_GRAB=$3 ./build/hgb 16 16 pack | tail -1
done
for nt in 1 0; do for g in hybrid cpu; do
  BK_PK_NT=$nt timeout 600 python bench.py --gather $g --steps 4 --warmup 3 --no-cpu-baseline --no-dbuf --no-profile > gpurun_out/pk_$g.json 2>gpurun_out/pk.err
  python3 -c "import json;d=json.load(open('gpurun_out/pk_$g.json'));print('nt=$nt grep $g', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'])" || tail -3 gpurun_out/pk.err
done; done
