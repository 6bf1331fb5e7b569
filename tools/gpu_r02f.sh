#!/bin/bash
# address mode (f2) + fused word count regression
mkdir -p gpurun_out
T=${TAG:-r02f}
timeout 900 python -m pytest tests/test_gpu_addr.py -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_addr.log 2>&1
tail -25 gpurun_out/${T}_addr.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_user.py tests/test_gpu_edge.py -q --timeout 600 --tb=short -p no:cacheprovider > gpurun_out/${T}_parity.log 2>&1
tail -5 gpurun_out/${T}_parity.log
