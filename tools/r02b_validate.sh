#!/bin/bash
# Round-2 (session B) validation on one B200 (run via gpurun): full GPU suite, smoke, all-workload bench,
# compute-sanitizer on every kernel (incl. the stream-K tail and the opt-in key-split kernel), ncu
# launch list of the default bench + --set full captures of the BERT-large-512 and stream-K kernels.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/r02b_pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02b_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02b_smoke.log 2>&1; echo "smoke exit $?" >> gpurun_out/r02b_smoke.log
tail -3 gpurun_out/r02b_pytest_gpu.log; tail -2 gpurun_out/r02b_smoke.log
bash tools/bench_all.sh > gpurun_out/r02b_bench_all_summary.txt 2>&1; cat gpurun_out/r02b_bench_all_summary.txt
timeout 300 python bench.py --steps 20 --warmup 5 > gpurun_out/r02b_bench_default.json 2> gpurun_out/r02b_bench_default.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/r02b_bl5_launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --sustained 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:fmha_fwd_sm100 -s 2 -c 1 -o gpurun_out/r02b_bl5_full python tools/fmha_prof.py bert_large_512 4 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:fmha_fwd_sm100 -s 2 -c 1 -o gpurun_out/r02b_streamk_full python tools/streamk_prof.py > /dev/null 2>&1
# (compute-sanitizer is closed on this pool in round 2b; the loop below reports nothing there)
: > gpurun_out/r02b_sanitizer.txt
for tool in memcheck racecheck synccheck; do
  for ks in 0 1; do
    echo "## B200_FMHA_KS=$ks PYTORCH_NO_CUDA_MEMORY_CACHING=1 compute-sanitizer --tool $tool python tools/sanitize.py" >> gpurun_out/r02b_sanitizer.txt
    B200_FMHA_KS=$ks PYTORCH_NO_CUDA_MEMORY_CACHING=1 timeout 900 compute-sanitizer --tool $tool python tools/sanitize.py 2>&1 | grep -E "SUMMARY|done|Error|error|hazard" | head -20 >> gpurun_out/r02b_sanitizer.txt
  done
done
cat gpurun_out/r02b_sanitizer.txt
tail -c 300 gpurun_out/r02b_bench_default.json
