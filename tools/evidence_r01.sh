cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
bash tools/bench_all.sh > gpurun_out/bench_all.log 2>&1
# launch lists (cold, serialised; shares only)
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/r01_mlp_fused_launches.csv python bench.py --workload mlp_fused --steps 5 --warmup 3 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/r01_splitkv_launches.csv python bench.py --workload decode_splitkv --steps 5 --warmup 3 > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r01_fmha_bl5_launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
# full captures
timeout 400 ncu --set full --clock-control none --import-source on -k regex:mlp_fused -s 3 -c 1 -o gpurun_out/r01_mlp_fused_full -f python bench.py --workload mlp_fused --steps 2 --warmup 3 > gpurun_out/mlp_ncu.log 2>&1
timeout 400 ncu --set full --clock-control none --import-source on -k regex:fmha_fwd -s 3 -c 1 -o gpurun_out/r01_splitkv_full -f python bench.py --workload decode_splitkv --steps 2 --warmup 3 > gpurun_out/splitkv_ncu.log 2>&1
echo evidence done
