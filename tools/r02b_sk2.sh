#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 300 python tools/sk_probe.py 2>&1 | tee gpurun_out/sk_probe2.txt
timeout 300 python -m pytest tests/test_streamk_gpu.py -x -q > gpurun_out/streamk_pytest.log 2>&1
echo "streamk pytest exit $?" >> gpurun_out/streamk_pytest.log
tail -4 gpurun_out/streamk_pytest.log
