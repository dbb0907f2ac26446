# Key-bias instance exponential-phase shape sweep (FMHA_BIAS_PRE_CHUNKS, FMHA_BIAS_POLY_CNT); default = (1, 2)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
L=paper_conf_asplos_hagedornfccgg23_b200/lib
for rep in 1 2; do for v in ${VARIANTS:-libb200fmha libb200fmha_b02 libb200fmha_b10 libb200fmha_b00 libb200fmha_b22 libb200fmha_b11 libb200fmha_b01 libb200fmha_b13}; do
  echo "== $v"; B200FMHA_LIB=$L/$v.so timeout 300 python tools/keybias_perf.py
done; done > gpurun_out/${OUT:-ab_bias_shape.txt} 2>&1
echo done
