#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q -k "causal or streamk or rescale" > gpurun_out/snake_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/snake_pytest.log; tail -3 gpurun_out/snake_pytest.log
bash tools/ab_env.sh gpt_causal 3 "B200_FMHA_SNAKE=0" "B200_FMHA_SNAKE=1" 2>&1 | tee gpurun_out/snake_ab.txt
