#!/bin/bash
# A/B of library variants in one session: tools/ab.sh <workload> <rounds> <variant>... ("" = default lib)
w=$1; r=$2; shift 2
for i in $(seq 1 $r); do
  for v in "$@"; do
    if [ "$v" = "default" ]; then lib="paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha.so"; else lib="paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_$v.so"; fi
    val=$(B200FMHA_LIB=$lib timeout 300 python bench.py --workload $w --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["value"], d["unit"], d["ms_per_step"])' 2>&1)
    echo "$w $v: $val"
  done
done
