# Race test of the idle-producer-warp fix (profiles/r02/race_r02.md): fault-free factorisations
# with the one-launch task-graph diagonal block on the high-priority panel stream and the
# BULK-copy update (forced), the round-2 kernel whose idle producer warps exit early (ABFT_WS=2x)
# vs the kernel whose idle producer warps stay resident until the consumers finish (default 2b).
# usage: bash tools/race_idle.sh [n] [nb] [reps (task-graph variants)] [reps (default path)] -> gpurun_out/race_idle_<n>.log
mkdir -p gpurun_out
n=${1:-32768}; nb=${2:-512}; reps=${3:-3}
out=gpurun_out/race_idle_$n.log
: > $out
run() {
  echo "=== $1" >> $out
  shift
  env "$@" REPS=$reps timeout 600 python tools/stress_v5.py $n $nb x 2>&1 | grep -E "status|Error|error" | cut -c1-200 >> $out
  echo "rc=$?" >> $out
}
reps2=${4:-$reps}
run tasks_G1_bulk_idle_exit_2x ABFT_CHOL=tasks ABFT_CHOL_G=1 ABFT_WS_FORCE_BULK=1 ABFT_WS=2x
run tasks_G1_bulk_idle_resident ABFT_CHOL=tasks ABFT_CHOL_G=1 ABFT_WS_FORCE_BULK=1
run tasks_G10_bulk_idle_exit_2x ABFT_CHOL=tasks ABFT_WS_FORCE_BULK=1 ABFT_WS=2x
run tasks_G10_bulk_idle_resident ABFT_CHOL=tasks ABFT_WS_FORCE_BULK=1
reps=$reps2
run default_idle_exit_2x ABFT_WS=2x
run default_idle_resident X=0
run default_idle_exit_2x_nchk3 ABFT_WS=2x ABFT_NCHK=3
run default_idle_resident_nchk3 ABFT_NCHK=3
