#!/bin/bash
# one-off (round 2, late): 32-B AVX2 packer copies (BK_PACK_CFG 7/8) vs the default (2), interleaved on one box
mkdir -p gpurun_out
T=${TAG:-r02p}
lscpu > gpurun_out/${T}_lscpu.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -k "packer" -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1
echo "packer tests rc=$? $(tail -1 gpurun_out/${T}_tests.log)"
for rep in 1 2; do
  for cfg in 2 7 8; do
    BK_PACK_CFG=$cfg timeout 900 python bench.py --steps 6 --warmup 3 --no-cpu-baseline --no-dbuf --no-profile --no-trace \
      > gpurun_out/${T}_grep_c${cfg}_$rep.json 2> gpurun_out/${T}_grep_c${cfg}_$rep.err
    python3 -c "import json;d=json.loads(open('gpurun_out/${T}_grep_c${cfg}_$rep.json').read().splitlines()[-1]);print('grep cfg=$cfg', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'])" || tail -3 gpurun_out/${T}_grep_c${cfg}_$rep.err
  done
done
for cfg in 2 7; do
  BK_PACK_CFG=$cfg timeout 900 python bench.py --workload kmer --steps 3 --warmup 3 --no-cpu-baseline --no-dbuf --no-profile --no-trace \
    > gpurun_out/${T}_kmer_c${cfg}.json 2> gpurun_out/${T}_kmer_c${cfg}.err
  python3 -c "import json;d=json.loads(open('gpurun_out/${T}_kmer_c${cfg}.json').read().splitlines()[-1]);print('kmer cfg=$cfg', d['value'], d['ms_per_step'], d['config']['chunks_cpu_assembled'])" || tail -3 gpurun_out/${T}_kmer_c${cfg}.err
done
