cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python tools/keybias_perf.py > gpurun_out/keybias_perf.txt 2>&1
bash tools/profile.sh r01_bl5_final
bash tools/profile.sh r01_bl384_final --workload bert_large_384
echo done
