cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTORCH_NO_CUDA_MEMORY_CACHING=1
for t in memcheck racecheck synccheck; do
  echo "## PYTORCH_NO_CUDA_MEMORY_CACHING=1 compute-sanitizer --tool $t python tools/sanitize.py  (every kernel incl. the key-bias instance with stride == seq_kv)"
  timeout 900 compute-sanitizer --tool $t python tools/sanitize.py 2>&1 | grep -v "^\s*$" | tail -4
  echo "$t exit ${PIPESTATUS[0]}"
done > gpurun_out/sanitizer.txt 2>&1
echo done
