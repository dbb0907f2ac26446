#!/bin/bash
# A/B bench runs over (library build, env) variants and workloads in one GPU session.
#   AB_VARIANTS="base: pdl0:B200_PDL=0 noturn@noturn:"  (name[@libsuffix]:ENV=VAL,...)
#   AB_WORKLOADS="bert_large_512 bert_large_varlen"
# Prints: workload variant value ms_per_step sm_mhz (two interleaved repetitions).
cd "$(dirname "$0")/.."
for rep in 1 2; do
  for wl in ${AB_WORKLOADS:-bert_large_512}; do
    for v in ${AB_VARIANTS:-base:}; do
      name=${v%%:*}; envs=${v#*:}
      lib=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha.so
      if [[ $name == *@* ]]; then lib=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_${name#*@}.so; fi
      (export B200FMHA_LIB=$lib; for kv in ${envs//,/ }; do export "$kv"; done
       timeout 300 python bench.py --workload "$wl" --steps ${AB_STEPS:-100} --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null |
         python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$wl', '$name', d['value'], d['ms_per_step'], d['clocks']['sm_mhz'])" ||
         echo "$wl $name FAILED")
    done
  done
done
