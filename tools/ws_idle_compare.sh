# Update kernel: idle producer warps resident (default 2b) vs exiting (2x, the earlier kernel):
# standalone SYRK and the whole C4 step (ABFT on/off, unprofiled).
mkdir -p gpurun_out
out=gpurun_out/ws_idle_compare.log
: > $out
for v in "resident X=0" "exit_2x ABFT_WS=2x"; do
  set -- $v; name=$1; shift
  echo "=== $name standalone" >> $out
  env "$@" timeout 300 python tools/gemm_bench.py 32256 512 >> $out 2>&1
  echo "=== $name C4 step" >> $out
  env "$@" timeout 600 python tools/time_arms.py 32768 512 3 >> $out 2>&1
done
