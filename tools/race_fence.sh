# Stage-release ordering experiment (profiles/r02/race_r02.md): fault-free C4 factorisations on the
# default path, the update/TRSM kernel without (ABFT_WS=2nf) and with (2b, now the default)
# fence.proxy.async before each stage release, in alternating blocks so box drift hits both arms
# alike. (The committed logs race_fence_*.log were taken when the fenced variant was named 2f and
# the unfenced one 2b: their arm names base_2b = unfenced, fence_2f = fenced.)
# NCHK3=1 / TASKS=1 add the three-checksum arms / the task-graph diagonal block with the bulk update
# usage: bash tools/race_fence.sh [n] [nb] [reps per block] [blocks] -> gpurun_out/race_fence_<n>.log
mkdir -p gpurun_out
n=${1:-32768}; nb=${2:-512}; reps=${3:-40}; blocks=${4:-4}
out=gpurun_out/race_fence_$n${TAG}.log
: > $out
run() {
  echo "=== $1" >> $out
  shift
  env "$@" REPS=$reps timeout 900 python tools/stress_v5.py $n $nb x 2>&1 | grep -E "status|Error|error" | cut -c1-200 >> $out
  echo "rc=$?" >> $out
}
for b in $(seq $blocks); do
  run nofence_2nf ABFT_WS=2nf
  run fence_2b ABFT_WS=2b
  if [ -n "$NCHK3" ]; then
    run nofence_2nf_nchk3 ABFT_WS=2nf ABFT_NCHK=3
    run fence_2b_nchk3 ABFT_WS=2b ABFT_NCHK=3
  fi
  if [ -n "$TASKS" ]; then
    run tasks_G1_nofence_2nf ABFT_WS=2nf ABFT_CHOL=tasks ABFT_CHOL_G=1
    run tasks_G1_fence_2b ABFT_WS=2b ABFT_CHOL=tasks ABFT_CHOL_G=1
  fi
done
awk '/^===/{name=$2; next} /status/{tot[name]++; if($5!=0||$3!=0)bad[name]++} END{for(k in tot) print k, bad[k]+0 "/" tot[k]}' $out | sort
