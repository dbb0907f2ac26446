#!/bin/bash
# ncu evidence for the bench workload (run via gpurun). $1 = tag, rest = extra bench args.
cd "$(dirname "$0")/.."
TAG=${1:-prof}; shift
mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e "$@" \
  > gpurun_out/${TAG}_launches.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fmha_fwd -s 3 -c 1 \
  -o gpurun_out/${TAG} -f python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e "$@" \
  > gpurun_out/${TAG}_full.log 2>&1
echo "profile exit $?"
tail -3 gpurun_out/${TAG}_full.log
