# Fault-free event rates of the DEFAULT path (recursive diagonal block, bulk-copy update with the
# producer tail): many back-to-back C4 factorisations with two and three checksum rows.
mkdir -p gpurun_out
out=gpurun_out/stress_rates.log
: > $out
for nc in 2 3; do
  echo "=== nchk=$nc" >> $out
  ABFT_NCHK=$nc REPS=${REPS:-25} timeout 900 python tools/stress_v5.py 32768 512 x 2>&1 | grep -E "status" | cut -c1-200 >> $out
done
