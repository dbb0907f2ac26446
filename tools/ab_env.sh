#!/bin/bash
# A/B of environment settings in one session: tools/ab_env.sh <workload> <rounds> "<ENV=..>" ...
w=$1; r=$2; shift 2
for i in $(seq 1 $r); do
  for e in "$@"; do
    val=$(env $e timeout 300 python bench.py --workload $w --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["value"], d["unit"], d["ms_per_step"])' 2>&1)
    echo "$w [$e]: $val"
  done
done
