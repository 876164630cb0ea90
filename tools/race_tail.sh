# The producer-tail fix (gemm.cu ws_body): the bulk-copy update with the task-graph diagonal block
# (which selects the LDGSTS producer by default; ABFT_WS_FORCE_BULK=1 keeps the bulk-copy one) and
# three-checksum fault-free runs, C4 and C5.
mkdir -p gpurun_out
out=gpurun_out/race_tail.log
: > $out
for cfg in "32768 512" "98304 1024"; do
  set -- $cfg
  echo "=== n=$1 tasks G=1 bulk-copy update" >> $out
  ABFT_WS_FORCE_BULK=1 ABFT_CHOL=tasks ABFT_CHOL_G=1 REPS=3 timeout 400 python tools/stress_v5.py $1 $2 x 2>&1 | grep -E "status" | cut -c1-160 >> $out
  echo "=== n=$1 tasks G=10 bulk-copy update" >> $out
  ABFT_WS_FORCE_BULK=1 ABFT_CHOL=tasks REPS=3 timeout 400 python tools/stress_v5.py $1 $2 x 2>&1 | grep -E "status" | cut -c1-160 >> $out
  echo "=== n=$1 nchk=3 default" >> $out
  ABFT_NCHK=3 REPS=5 timeout 400 python tools/stress_v5.py $1 $2 x 2>&1 | grep -E "status" | cut -c1-160 >> $out
done
