#!/bin/bash
# Round-2 session B: FMHA_SUMCHECK variant -- GPU suite against it, then A/B vs the default build.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
V=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_sumchk.so
B200FMHA_LIB=$V timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/sumchk_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/sumchk_pytest.log
tail -3 gpurun_out/sumchk_pytest.log
for w in bert_large_512 bert_large_384 bert_large_varlen; do
  bash tools/ab.sh $w 3 default sumchk
done 2>&1 | tee gpurun_out/sumchk_ab.txt
