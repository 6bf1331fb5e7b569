#!/bin/bash
# Re-entry confirmation: build on the box, smoke, GPU parity suite, default bench line.
mkdir -p gpurun_out
TAG=${TAG:-r01c}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,pcie.link.gen.current,pcie.link.width.current --format=csv > gpurun_out/${TAG}_smi.txt 2>&1
nproc >> gpurun_out/${TAG}_smi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; tail -1 gpurun_out/${TAG}_smoke.log
timeout 1200 python -m pytest tests -m gpu -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -2 gpurun_out/${TAG}_gpu_tests.log
timeout 900 python bench.py > gpurun_out/${TAG}_bench_grep.json 2> gpurun_out/${TAG}_bench_grep.err
python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_grep.json'));print('grep', d['value'], d['ms_per_step'], d['link']['frac'], d['roofline']['frac'], d['clocks'])" || tail -5 gpurun_out/${TAG}_bench_grep.err
