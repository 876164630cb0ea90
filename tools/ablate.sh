# ABFT overhead attribution at C4: one process per ablation mask (ABFT_DEV_ABLATE).
mkdir -p gpurun_out
out=gpurun_out/ablate_${N:-32768}.jsonl
: > $out
for m in 0 2 4 8 6 22 23 31; do
  ABFT_DEV_ABLATE=$m timeout 600 python tools/time_arms.py ${N:-32768} ${NB:-512} ${PAIRS:-3} >> $out 2>> gpurun_out/ablate.err
done
