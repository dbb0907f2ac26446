#!/bin/bash
# Round-2 session B: stream-K tail -- GPU suite (incl. test_streamk_gpu.py), then A/B on BERT-large-384.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_streamk_gpu.py -x -q > gpurun_out/streamk_pytest.log 2>&1
echo "streamk pytest exit $?" >> gpurun_out/streamk_pytest.log
tail -15 gpurun_out/streamk_pytest.log
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
for i in 1 2 3; do
  for sk in off on; do
    v=$(timeout 300 python bench.py --workload bert_large_384 --stream-k $sk --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(d["value"], d["ms_per_step"], d["config"]["kernel"])')
    echo "bert_large_384 stream-k=$sk: $v"
  done
done 2>&1 | tee gpurun_out/streamk_ab.txt
