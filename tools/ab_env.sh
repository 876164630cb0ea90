# Same-box A/B of a library knob (one process per run, alternating): tools/time_arms.py at C2, C3, C4
# usage: bash tools/ab_env.sh "ENV_A" "ENV_B" [reps] -> gpurun_out/ab_env.jsonl
mkdir -p gpurun_out
A=${1:-X=0}; B=${2:-X=1}; reps=${3:-2}
for r in $(seq $reps); do
  for cfg in "4096 256" "16384 512" "32768 512"; do
    env $A timeout 600 python tools/time_arms.py $cfg 5 >> gpurun_out/ab_env.jsonl 2>> gpurun_out/ab_env.err
    env $B timeout 600 python tools/time_arms.py $cfg 5 >> gpurun_out/ab_env.jsonl 2>> gpurun_out/ab_env.err
  done
done
