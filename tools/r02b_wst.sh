#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
V=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_wst.so
B200FMHA_LIB=$V timeout 600 python -m pytest tests/test_gemm_gpu.py tests/test_layer_gpu.py -x -q > gpurun_out/wst_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/wst_pytest.log; tail -2 gpurun_out/wst_pytest.log
for w in mlp lstm_cell bert_layer; do bash tools/ab.sh $w 3 default wst; done 2>&1 | tee gpurun_out/wst_ab.txt
B200FMHA_LIB=$V python tools/gemm_compare.py 2>&1 | tee -a gpurun_out/wst_ab.txt
