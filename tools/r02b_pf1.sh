#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
V=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_pf1.so
for w in bert_base_pad bert_large_512 bert_large_384 gpt_causal; do bash tools/ab.sh $w 3 default pf1; done 2>&1 | tee gpurun_out/pf1_ab.txt
for i in 1 2; do
  python tools/shard_time.py 2>&1 | sed 's/^/default /'
  B200FMHA_LIB=$V python tools/shard_time.py 2>&1 | sed 's/^/pf1 /'
done | tee -a gpurun_out/pf1_ab.txt
B200FMHA_LIB=$V timeout 900 python -m pytest tests/test_fmha_gpu.py tests/test_streamk_gpu.py tests/test_keybias_gpu.py -x -q > gpurun_out/pf1_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/pf1_pytest.log; tail -2 gpurun_out/pf1_pytest.log
