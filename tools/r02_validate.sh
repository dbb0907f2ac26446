#!/bin/bash
# Round-2 validation on one B200 (run via gpurun): full GPU suite, smoke, compute-sanitizer on every
# kernel (incl. the opt-in key-split kernel), results under gpurun_out/.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/r02_pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_smoke.log 2>&1; echo "smoke exit $?" >> gpurun_out/r02_smoke.log
: > gpurun_out/r02_sanitizer.txt
for tool in memcheck racecheck synccheck; do
  for ks in 0 1; do
    echo "## B200_FMHA_KS=$ks PYTORCH_NO_CUDA_MEMORY_CACHING=1 compute-sanitizer --tool $tool python tools/sanitize.py" >> gpurun_out/r02_sanitizer.txt
    B200_FMHA_KS=$ks PYTORCH_NO_CUDA_MEMORY_CACHING=1 timeout 900 compute-sanitizer --tool $tool python tools/sanitize.py 2>&1 | grep -E "SUMMARY|done|Error|error|hazard" | head -20 >> gpurun_out/r02_sanitizer.txt
  done
done
tail -3 gpurun_out/r02_pytest_gpu.log; cat gpurun_out/r02_smoke.log | tail -2; cat gpurun_out/r02_sanitizer.txt
# ncu: launch list of the default bench command and one --set full capture of the BERT-large-512 kernel
ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/r02_bl5_launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --sustained 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:fmha_fwd_sm100 -s 2 -c 1 -o gpurun_out/r02_bl5_full python tools/fmha_prof.py bert_large_512 4 > /dev/null 2>&1
timeout 300 python bench.py --steps 20 --warmup 5 > gpurun_out/r02_bench_default.json 2> gpurun_out/r02_bench_default.err
tail -c 400 gpurun_out/r02_bench_default.json
