cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export B200FMHA_LIB=paper_conf_asplos_hagedornfccgg23_b200/lib/libb200fmha_hc.so
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pt_full.log 2>&1; echo "pytest exit $?" >> gpurun_out/pt_full.log
tail -3 gpurun_out/pt_full.log
unset B200FMHA_LIB
for w in ${WL:-bert_large_512 bert_large_384 bert_base_pad}; do AB_ARGS="--workload $w" timeout 600 bash tools/ab.sh ${AB} 2>&1 | sed "s/^/$w /"; done
