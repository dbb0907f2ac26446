cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
L=paper_conf_asplos_hagedornfccgg23_b200/lib
for rep in 1 2 3; do for v in libb200fmha libb200fmha_orig; do
  echo "== $v"; B200FMHA_LIB=$L/$v.so timeout 300 python tools/keybias_perf.py
done; done > gpurun_out/ab_bias.txt 2>&1
timeout 900 python -m pytest tests/test_keybias_gpu.py tests/test_varlen_gpu.py -q > gpurun_out/pytest_bias.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_bias.log
echo done
