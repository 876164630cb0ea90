# Race bisection of the warp-specialised update kernel: fault-free C5 factorisations
# with the one-launch diagonal block on the high-priority panel stream (the known trigger), one
# process per variant (the library reads its knobs once). A clean run raises no event.
mkdir -p gpurun_out
out=gpurun_out/race_matrix.log
: > $out
run() {
  echo "=== $1" >> $out
  shift
  env "$@" ABFT_CHOL=tasks ABFT_CHOL_G=1 REPS=${REPS:-2} timeout 300 python tools/stress_v5.py ${N:-98304} ${NB:-1024} x >> $out 2>&1
  echo "rc=$?" >> $out
}
run default X=0
run fence_consumer ABFT_WS_DBG=1
run producer_tail ABFT_WS_DBG=2
run tail_idle_resident ABFT_WS_DBG=6
run c_preload_cg ABFT_WS_DBG=8
run no_l2_prefetch ABFT_WS_PF=0
run ldgsts_producer ABFT_WS=2l
