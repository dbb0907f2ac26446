cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1
timeout 300 python bench.py --workload bert_large_varlen --steps 100 --warmup 5 --no-cpu-baseline > gpurun_out/bench_varlen.json 2>/dev/null
timeout 300 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
echo done
