# Update-kernel producer comparison: bulk-copy (default) vs LDGSTS (ABFT_WS=2l), standalone SYRK and
# the whole C4 step (ABFT on/off, unprofiled), with and without the task-graph diagonal block.
mkdir -p gpurun_out
out=gpurun_out/ws_compare.log
: > $out
for v in "bulk X=0" "ldgsts ABFT_WS=2l"; do
  set -- $v; name=$1; shift
  echo "=== $name standalone" >> $out
  env "$@" timeout 300 python tools/gemm_bench.py 32256 512 >> $out 2>&1
  env "$@" timeout 300 python tools/gemm_bench.py 16384 512 >> $out 2>&1
  echo "=== $name C4 step" >> $out
  env "$@" timeout 600 python tools/time_arms.py 32768 512 3 >> $out 2>&1
  echo "=== $name C4 step, tasks diagonal block" >> $out
  env "$@" ABFT_CHOL=tasks timeout 600 python tools/time_arms.py 32768 512 3 >> $out 2>&1
done
