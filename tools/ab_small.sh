# Same-box A/B of two in-tree builds at C2 (graph mode, tools/c2_ablate.py) and C4 (tools/time_arms.py)
mkdir -p gpurun_out
A=${1:-X=0}; B=${2:-X=1}; reps=${3:-3}
for r in $(seq $reps); do
  env $A timeout 300 python tools/c2_ablate.py 4096 256 | sed "s/^{/{\"env\": \"$A\", /" >> gpurun_out/ab_small.jsonl
  env $B timeout 300 python tools/c2_ablate.py 4096 256 | sed "s/^{/{\"env\": \"$B\", /" >> gpurun_out/ab_small.jsonl
done
env $A timeout 600 python tools/time_arms.py 32768 512 5 >> gpurun_out/ab_env.jsonl
env $B timeout 600 python tools/time_arms.py 32768 512 5 >> gpurun_out/ab_env.jsonl
