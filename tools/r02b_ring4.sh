#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
V=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_ring4.so
D=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha.so
bash tools/ab.sh gpt_causal 3 default ring4 2>&1 | tee gpurun_out/ring4_ab.txt
for i in 1 2; do
  B200FMHA_LIB=$D timeout 200 python tools/shape_time.py default
  B200FMHA_LIB=$V timeout 200 python tools/shape_time.py ring4
done 2>&1 | tee -a gpurun_out/ring4_ab.txt
B200FMHA_LIB=$V timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/ring4_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/ring4_pytest.log; tail -2 gpurun_out/ring4_pytest.log
