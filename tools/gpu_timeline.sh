#!/bin/bash
# Per-stage event timelines (BK_TIMELINE CSV) of the profiled pass of bench lines, plus the tests the change touches.
mkdir -p gpurun_out
TAG=${TAG:-r01t}
[ -n "$NOTEST" ] || timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "partition or cid or kmeans or profiled" --timeout 600 -p no:cacheprovider > gpurun_out/${TAG}_tests.log 2>&1; tail -1 gpurun_out/${TAG}_tests.log
for w in ${WS:-partition wordcount}; do
  rm -f gpurun_out/${TAG}_tl_$w.csv
  BK_TIMELINE=gpurun_out/${TAG}_tl_$w.csv timeout 600 python bench.py --workload $w --no-cpu-baseline --no-dbuf $ARGS > gpurun_out/${TAG}_bench_$w.json 2> gpurun_out/${TAG}_bench_$w.err
  python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_$w.json'));print('$w', d['value'], d['ms_per_step'], d['link']['frac'], d['overlap'], d['roofline']['kernel'], round(d['roofline']['frac'],4))" || tail -5 gpurun_out/${TAG}_bench_$w.err
done
