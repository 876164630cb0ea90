# The shipped (fenced) update pipeline under the configurations that exposed the stage-release race
# (profiles/r02/race_r02.md): fault-free factorisations, one process per block.
# usage: bash tools/race_fixed.sh [n] [nb] [reps per block] [blocks] -> gpurun_out/race_fixed_<n>.log
mkdir -p gpurun_out
n=${1:-32768}; nb=${2:-512}; reps=${3:-40}; blocks=${4:-4}
out=gpurun_out/race_fixed_$n${TAG}.log
: > $out
run() {
  echo "=== $1" >> $out
  shift
  env "$@" REPS=$reps timeout 900 python tools/stress_v5.py $n $nb x 2>&1 | grep -E "status|Error|error" | cut -c1-200 >> $out
  echo "rc=$?" >> $out
}
for b in $(seq $blocks); do
  run default_recursive X=0
  run tasks_G10 ABFT_CHOL=tasks
  run tasks_G1 ABFT_CHOL=tasks ABFT_CHOL_G=1
  run default_recursive_nchk3 ABFT_NCHK=3
done
awk '/^===/{name=$2; next} /status/{tot[name]++; if($5!=0||$3!=0)bad[name]++} END{for(k in tot) print k, bad[k]+0 "/" tot[k]}' $out | sort
