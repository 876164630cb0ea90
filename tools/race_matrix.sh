# Race bisection of the warp-specialised update kernel: fault-free factorisations,
# one process per variant (the library reads its knobs once). A clean run raises no event.
# usage: bash tools/race_matrix.sh [n] [nb] [reps] -> gpurun_out/race_matrix_<n>.log
mkdir -p gpurun_out
n=${1:-98304}; nb=${2:-1024}; reps=${3:-3}
out=gpurun_out/race_matrix_$n.log
: > $out
run() {
  echo "=== $1" >> $out
  shift
  env "$@" REPS=$reps timeout 400 python tools/stress_v5.py $n $nb x 2>&1 | grep -E "status|Error|error" | cut -c1-200 >> $out
  echo "rc=$?" >> $out
}
run default_recursive_highprio X=0
run tasks_G1 ABFT_CHOL=tasks ABFT_CHOL_G=1
run tasks_G10 ABFT_CHOL=tasks
run tasks_G1_normal_prio ABFT_CHOL=tasks ABFT_CHOL_G=1 ABFT_P_PRIO=0
run tasks_G1_ldgsts ABFT_CHOL=tasks ABFT_CHOL_G=1 ABFT_WS=2l
run tasks_G1_cp_async_gemm ABFT_CHOL=tasks ABFT_CHOL_G=1 ABFT_GEMM_VARIANT=2
run recursive_nofuse ABFT_NOFUSE=1
