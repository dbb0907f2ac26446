# Varlen instance exponential-phase shape sweep (FMHA_VARLEN_PRE_CHUNKS, FMHA_VARLEN_POLY_CNT); default = dense (1, 2)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
AB_STEPS=100 AB_WORKLOADS="bert_large_varlen" AB_VARIANTS="${VARIANTS:-base: v00@v00: v01@v01: v02@v02: v11@v11: v22@v22: v21@v21: v03@v03:}" bash tools/ab_env.sh > gpurun_out/${OUT:-ab_varlen_shape.txt} 2>&1
echo done
