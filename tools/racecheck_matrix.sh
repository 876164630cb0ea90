# racecheck of the update GEMM alone (M = 2304: the warp-specialised path) under each operand-
# staging scheme: does the tool see the mbarrier synchronisation of each?
mkdir -p gpurun_out
out=gpurun_out/racecheck_matrix.log
: > $out
for v in "bulk_copy_default X=0" "ldgsts_producer ABFT_WS=2l" "cp_async_syncthreads ABFT_GEMM_VARIANT=2"; do
  set -- $v
  name=$1; shift
  echo "=== $name" >> $out
  env "$@" timeout 900 compute-sanitizer --tool racecheck --print-limit 3 tools/bin/sanitize_driver 2304 256 gemm 2>&1 | grep -E "Error:|Warning:|SUMMARY|hazards\]|gemm_nt|OK|FAIL" | cut -c1-220 | head -12 >> $out
done
