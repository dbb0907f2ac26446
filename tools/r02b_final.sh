#!/bin/bash
# Round-2b final validation of the committed build (run via gpurun): GPU suite, smoke, all-workload bench,
# default bench line, ncu launch list + --set full of the BERT-large-512 kernel and of the MLP GELU GEMM.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/r02c_pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02c_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02c_smoke.log 2>&1; echo "smoke exit $?" >> gpurun_out/r02c_smoke.log
tail -2 gpurun_out/r02c_pytest_gpu.log; tail -2 gpurun_out/r02c_smoke.log
bash tools/bench_all.sh > gpurun_out/r02c_bench_all_summary.txt 2>&1; cat gpurun_out/r02c_bench_all_summary.txt
cp gpurun_out/bench_all.jsonl gpurun_out/r02c_bench_all.jsonl
timeout 300 python bench.py > gpurun_out/r02c_bench_default.json 2> gpurun_out/r02c_bench_default.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/r02c_bl5_launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --sustained 0 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:fmha_fwd_sm100 -s 2 -c 1 -o gpurun_out/r02c_bl5_full python tools/fmha_prof.py bert_large_512 4 > /dev/null 2>&1
ncu --set full --clock-control none -k regex:gemm_bias_act_2sm_kernel -c 2 -o gpurun_out/r02c_gemm_full python tools/gemm_prof.py 1 > /dev/null 2>&1
tail -c 600 gpurun_out/r02c_bench_default.json
