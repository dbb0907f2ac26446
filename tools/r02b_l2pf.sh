#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
V=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_l2pf.so
for w in bert_large_512 bert_large_384 gpt_causal bert_base_pad; do bash tools/ab.sh $w 3 default l2pf; done 2>&1 | tee gpurun_out/l2pf_ab.txt
B200FMHA_LIB=$V timeout 900 python -m pytest tests/test_fmha_gpu.py tests/test_streamk_gpu.py -x -q > gpurun_out/l2pf_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/l2pf_pytest.log; tail -2 gpurun_out/l2pf_pytest.log
