#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-r01g}
timeout 900 python -m pytest tests -m gpu -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${TAG}_gpu_tests.log 2>&1
tail -4 gpurun_out/${TAG}_gpu_tests.log
timeout 600 python bench.py > gpurun_out/${TAG}_bench_grep.json 2> gpurun_out/${TAG}_bench_grep.err
python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_grep.json'));print('grep', d['value'], d['ms_per_step'], d['link'], d['roofline'], d.get('cpu_baseline'), d['clocks'])" || tail -5 gpurun_out/${TAG}_bench_grep.err
for w in wordcount groupby kmeans partition; do
  timeout 600 python bench.py --workload $w --steps 3 --warmup 3 > gpurun_out/${TAG}_bench_$w.json 2> gpurun_out/${TAG}_bench_$w.err
  python3 -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_$w.json'));print('$w', d['value'], d['ms_per_step'], d['link']['frac'], d['stages_ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], d.get('cpu_baseline',{}).get('value'))" || tail -5 gpurun_out/${TAG}_bench_$w.err
done
BK_BENCH_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --gib 2 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_grep_2rank.json 2> gpurun_out/${TAG}_bench_grep_2rank.err
tail -c 600 gpurun_out/${TAG}_bench_grep_2rank.json; tail -3 gpurun_out/${TAG}_bench_grep_2rank.err
BK_BENCH_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 2 --workload partition --gib 1 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_part_2rank.json 2> gpurun_out/${TAG}_bench_part_2rank.err
tail -c 400 gpurun_out/${TAG}_bench_part_2rank.json; tail -3 gpurun_out/${TAG}_bench_part_2rank.err
