# Chunked task-graph diagonal block, G = 1 and 2 CTAs per chunk: stress + timing.
mkdir -p gpurun_out
out=gpurun_out/race_chunks2.log
: > $out
for G in 1 2; do
  echo "=== timing C4 / C3 / C2, chunked tasks G=$G + bulk" >> $out
  for cfg in "32768 512 3" "16384 512 5" "4096 256 5"; do
    set -- $cfg
    ABFT_WS_FORCE_BULK=1 ABFT_CHOL=tasks ABFT_CHOL_G=$G ABFT_CHOL_CHUNKS=16 timeout 600 python tools/time_arms.py $1 $2 $3 2>&1 | cut -c1-330 >> $out
  done
  echo "=== n=98304 tasks G=$G chunks=16 bulk" >> $out
  ABFT_WS_FORCE_BULK=1 ABFT_CHOL=tasks ABFT_CHOL_G=$G ABFT_CHOL_CHUNKS=16 REPS=6 timeout 700 python tools/stress_v5.py 98304 1024 x 2>&1 | grep -E "status|Error" | cut -c1-160 >> $out
  echo "=== n=32768 tasks G=$G chunks=8 bulk" >> $out
  ABFT_WS_FORCE_BULK=1 ABFT_CHOL=tasks ABFT_CHOL_G=$G ABFT_CHOL_CHUNKS=8 REPS=12 timeout 700 python tools/stress_v5.py 32768 512 x 2>&1 | grep -E "status|Error" | cut -c1-160 >> $out
done
