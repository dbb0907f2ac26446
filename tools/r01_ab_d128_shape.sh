# D = 128 exponential-phase shape sweep (FMHA_PRE_CHUNKS for D = 128, FMHA_POLY_CNT128); default = (0, 0)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
AB_STEPS=50 AB_WORKLOADS="gpt_causal" AB_VARIANTS="base: d01@d01: d02@d02: d10@d10: d11@d11: d20@d20:" bash tools/ab_env.sh > gpurun_out/ab_d128_shape.txt 2>&1
echo done
