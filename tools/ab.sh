#!/bin/bash
# A/B the bench between library builds in one GPU session: tools/ab.sh name1 name2 ... (lib/libb200fmha_<name>.so)
cd "$(dirname "$0")/.."
for rep in 1 2; do
  for n in "$@"; do
    B200FMHA_LIB=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_$n.so python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e ${AB_ARGS} | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$n', d['value'], d['ms_per_step'], d['clocks']['sm_mhz'])"
  done
done
