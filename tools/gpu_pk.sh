#!/bin/bash
./build/cpu_gather_probe 16 | tail -3
for cfg in "1 16 16384" "0 16 16384" "1 0 16384" "0 0 16384" "1 16 262144" "0 0 262144" "1 32 65536"; do set -- $cfg
  echo "nt=$1 pf=$2 grab=$3"; BK_PK_NT=$1 BK_PK_PF=$2 BK_PK_GRAB=$3 ./build/hgb 16 16 pack | tail -1
done
