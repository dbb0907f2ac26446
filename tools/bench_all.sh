#!/bin/bash
# All BASELINE.json workloads on one GPU (run via gpurun); JSON lines -> gpurun_out/bench_all.jsonl
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
: > gpurun_out/bench_all.jsonl
for w in bert_large_512 bert_large_384 bert_base_pad gpt_causal tiny mlp bert_large_varlen bert_layer lstm_cell mlp_fused mlp_fused_w64 decode_splitkv; do
  timeout 300 python bench.py --workload $w --steps ${STEPS:-50} --warmup 5 --no-cpu-baseline --no-e2e \
    >> gpurun_out/bench_all.jsonl 2> gpurun_out/bench_all_$w.err || echo "{\"workload\": \"$w\", \"error\": true}" >> gpurun_out/bench_all.jsonl
done
timeout 300 python bench.py --steps 50 --warmup 5 > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
cat gpurun_out/bench_all.jsonl | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); print(d.get('config',{}).get('workload', d.get('workload')), d.get('value'), d.get('ms_per_step'), d.get('roofline',{}).get('frac'))"
