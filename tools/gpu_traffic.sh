#!/bin/bash
# One ncu --set full capture of the roofline kernel of each bench line whose dominant stage is a
# kernel (not a copy-engine DMA), with the bench JSON of the same command (units per launch):
# tools/traffic_json.py turns them into profiles/r0N_traffic.json, which bench.py scales into
# roofline.traffic.
mkdir -p gpurun_out
TAG=${TAG:-r02x}
B="python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-dbuf --no-profile --no-trace"
cap() {  # name kernel-regex skip bench-args
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$2" -s $3 -c 1 \
      -o gpurun_out/${TAG}_tr_$1 $B $4 > gpurun_out/${TAG}_tr_$1.json 2> gpurun_out/${TAG}_tr_$1.err
  echo "$1 rc=$? $(tail -c 200 gpurun_out/${TAG}_tr_$1.json | tr -d '\n' | tail -c 80)"
}
cap grep "k_gather_field" 6 "--workload grep --gib 4 --zc-share 1000"
cap groupby_sparse "k_gather_field" 6 "--workload groupby_sparse --gib 4 --zc-share 1000"
cap wordcount "k_wc_fused" 3 "--workload wordcount"
# k-mers: three kernels per chunk, per-kernel DRAM bytes in profiles/r02_kmer.md (no single roofline kernel)
