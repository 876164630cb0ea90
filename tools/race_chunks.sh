# Is it the LIFETIME of the high-priority CTAs? The task-graph diagonal block split into short
# launches at step boundaries (ABFT_CHOL_CHUNKS) next to the bulk-copy update, C4 and C5.
mkdir -p gpurun_out
out=gpurun_out/race_chunks.log
: > $out
for cfg in "32768 512 8" "98304 1024 16"; do
  set -- $cfg
  for G in 1 10; do
    echo "=== n=$1 tasks G=$G chunks=$3 bulk-copy update" >> $out
    ABFT_WS_FORCE_BULK=1 ABFT_CHOL=tasks ABFT_CHOL_G=$G ABFT_CHOL_CHUNKS=$3 REPS=4 timeout 500 python tools/stress_v5.py $1 $2 x 2>&1 | grep -E "status|Error" | cut -c1-160 >> $out
  done
done
echo "=== timing C4 / C3, chunked tasks + bulk" >> $out
ABFT_WS_FORCE_BULK=1 ABFT_CHOL=tasks ABFT_CHOL_CHUNKS=8 timeout 600 python tools/time_arms.py 32768 512 3 >> $out 2>&1
ABFT_WS_FORCE_BULK=1 ABFT_CHOL=tasks ABFT_CHOL_CHUNKS=8 timeout 600 python tools/time_arms.py 16384 512 3 >> $out 2>&1
