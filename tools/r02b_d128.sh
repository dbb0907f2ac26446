#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
V=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_${1:-sumchk128}.so
D=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha.so
for i in 1 2; do
  B200FMHA_LIB=$D timeout 200 python tools/shape_time.py default
  B200FMHA_LIB=$V timeout 200 python tools/shape_time.py ${1:-sumchk128}
done 2>&1 | tee gpurun_out/d128_ab.txt
B200FMHA_LIB=$V timeout 900 python -m pytest tests -m gpu -x -q ${PYTEST_K} > gpurun_out/d128_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/d128_pytest.log; tail -3 gpurun_out/d128_pytest.log
