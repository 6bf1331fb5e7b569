#!/bin/bash
# Look-ahead stage 1 for ZC plans: parity (ZC paths, graphs, delays) + A/B bench (BK_NO_LOOKAHEAD).
mkdir -p gpurun_out
TAG=${TAG:-r01la}
timeout 900 python -m pytest tests -m gpu -q -x -k "zc or wordcount or repeated or delays or invariance or layout or edge or user or kmer or pattern or profiled" -p no:cacheprovider > gpurun_out/${TAG}_tests.log 2>&1; tail -1 gpurun_out/${TAG}_tests.log
for r in 1 2; do for v in 0 1; do
  if [ $v = 1 ]; then export BK_NO_LOOKAHEAD=1; else unset BK_NO_LOOKAHEAD; fi
  timeout 300 python bench.py --workload wordcount --steps 30 --warmup 5 --no-cpu-baseline --no-dbuf > gpurun_out/${TAG}_wc_$v.json 2>/dev/null
  python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_wc_$v.json'));print('wc nolookahead=$v', d['value'], d['ms_per_step'])"
done; done
unset BK_NO_LOOKAHEAD
for sl in 4 16; do timeout 300 python bench.py --workload wordcount --steps 30 --warmup 5 --slots $sl --no-cpu-baseline --no-dbuf > gpurun_out/${TAG}_wc_s$sl.json 2>/dev/null
  python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_wc_s$sl.json'));print('wc slots $sl', d['value'], d['ms_per_step'])"; done
