#!/bin/bash
# round 2: new tests first, then the whole GPU suite, then the default bench line
mkdir -p gpurun_out
T=${TAG:-r02a}
timeout 900 python -m pytest tests/test_gpu_api_state.py tests/test_gpu_merge.py tests/test_gpu_ranks_parity.py -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_new.log 2>&1
tail -30 gpurun_out/${T}_new.log
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 --tb=short -p no:cacheprovider > gpurun_out/${T}_gpu_tests.log 2>&1
tail -15 gpurun_out/${T}_gpu_tests.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/${T}_bench_grep.json 2> gpurun_out/${T}_bench_grep.err
tail -c 600 gpurun_out/${T}_bench_grep.json; tail -3 gpurun_out/${T}_bench_grep.err
