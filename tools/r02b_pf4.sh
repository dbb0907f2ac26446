#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for w in bert_base_pad bert_large_512 bert_large_384 gpt_causal; do bash tools/ab.sh $w 2 pf1s pf1 pf4; done 2>&1 | tee gpurun_out/pf4_ab.txt
for v in pf1s pf1 pf4; do B200FMHA_LIB=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_$v.so python tools/shard_time.py 2>&1 | sed "s/^/$v /" | tail -1; done | tee -a gpurun_out/pf4_ab.txt
