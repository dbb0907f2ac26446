#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for v in default skabl1 skabl3; do
  if [ $v = default ]; then lib=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha.so; else lib=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_$v.so; fi
  echo "== $v"; B200FMHA_LIB=$lib timeout 300 python tools/sk_probe.py
done 2>&1 | tee gpurun_out/sk_probe.txt
