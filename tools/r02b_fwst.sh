#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
V=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_fwst.so
for w in bert_base_pad bert_large_384 bert_large_512 gpt_causal; do bash tools/ab.sh $w 3 default fwst; done 2>&1 | tee gpurun_out/fwst_ab.txt
B200FMHA_LIB=$V timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/fwst_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/fwst_pytest.log; tail -2 gpurun_out/fwst_pytest.log
