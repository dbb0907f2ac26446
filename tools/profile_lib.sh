#!/bin/bash
# ncu --set full of the FMHA kernel for a given library build: tools/profile_lib.sh <name> [bench args]
cd "$(dirname "$0")/.."
n=$1; shift
B200FMHA_LIB=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_$n.so timeout 600 ncu --set full --clock-control none --import-source on -k regex:fmha_fwd -s 3 -c 1 -o gpurun_out/prof_$n -f python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e "$@" > gpurun_out/prof_$n.log 2>&1
echo "profile $n exit $?"
