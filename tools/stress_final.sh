# Fault-free stress of the shipped configuration (task-graph diagonal block, fenced bulk-copy
# update): back-to-back C4 and C5 factorisations; every run must end with status 0 and no event.
mkdir -p gpurun_out
REPS=${C4_REPS:-150} timeout 1200 python tools/stress_v5.py 32768 512 x 2>&1 | grep -E "status" > gpurun_out/stress_c4.log
REPS=${C5_REPS:-12} timeout 1200 python tools/stress_v5.py 98304 1024 x 2>&1 | grep -E "status" > gpurun_out/stress_c5.log
for f in gpurun_out/stress_c4.log gpurun_out/stress_c5.log; do
  echo "$f: $(grep -c status $f) runs, $(awk '$3!=0||$5!=0' $f | wc -l) with a non-zero status or events"
done
