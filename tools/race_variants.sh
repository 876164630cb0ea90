# Which change removed the stage-release failures (profiles/r02/race_r02.md)? Fault-free C4
# factorisations with the one-launch task-graph diagonal block (G = 1: longest-lived high-priority
# CTAs) and the bulk-copy update in three variants, alternating blocks on one box:
#   2x  : round-2 kernel — idle producer warps exit right after setmaxnreg.dec, no consumer fence
#   2nf : idle producer warps stay resident, no consumer fence
#   2b  : resident + consumer fence.proxy.async (the shipped kernel)
# usage: bash tools/race_variants.sh [n] [nb] [reps per block] [blocks] -> gpurun_out/race_variants_<n>.log
mkdir -p gpurun_out
n=${1:-32768}; nb=${2:-512}; reps=${3:-30}; blocks=${4:-2}
out=gpurun_out/race_variants_$n.log
: > $out
run() {
  echo "=== $1" >> $out
  shift
  env "$@" REPS=$reps timeout 900 python tools/stress_v5.py $n $nb x 2>&1 | grep -E "status|Error|error" | cut -c1-200 >> $out
  echo "rc=$?" >> $out
}
for b in $(seq $blocks); do
  run tasks_G1_2x_idle_exit_nofence ABFT_WS=2x ABFT_CHOL=tasks ABFT_CHOL_G=1
  run tasks_G1_2nf_resident_nofence ABFT_WS=2nf ABFT_CHOL=tasks ABFT_CHOL_G=1
  run tasks_G1_2b_resident_fence ABFT_WS=2b ABFT_CHOL=tasks ABFT_CHOL_G=1
done
awk '/^===/{name=$2; next} /status/{tot[name]++; if($5!=0||$3!=0)bad[name]++} END{for(k in tot) print k, bad[k]+0 "/" tot[k]}' $out | sort
