#!/bin/bash
# host packer prefetch sweep (host-only; the GPU box's 16 vCPUs): build/hgb <GiB> <threads> pack
mkdir -p gpurun_out
T=${TAG:-r02r}
for cfg in "16 0 0" "16 0 1" "32 0 1" "16 64 1" "16 128 1" "8 64 1" "32 128 1" "64 0 1"; do set -- $cfg
  BK_PACK_PF=$1 BK_PACK_PF2=$2 BK_PACK_PFEND=$3 timeout 300 ./build/hgb 16 16 pack > gpurun_out/${T}_hgb_$1_$2_$3.txt 2>&1
  echo "pf=$1 pf2=$2 end=$3 $(tail -1 gpurun_out/${T}_hgb_$1_$2_$3.txt)"
done
