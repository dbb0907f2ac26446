#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
V=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_lpt.so
B200FMHA_LIB=$V timeout 900 python -m pytest tests/test_varlen_gpu.py tests/test_layer_gpu.py tests/test_rescale_gpu.py -x -q > gpurun_out/lpt_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/lpt_pytest.log; tail -2 gpurun_out/lpt_pytest.log
for w in bert_large_varlen bert_layer; do bash tools/ab.sh $w 3 default lpt; done 2>&1 | tee gpurun_out/lpt_ab.txt
