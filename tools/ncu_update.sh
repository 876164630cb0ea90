# ncu --set full of the k=0 trailing update (b) at C4 under three ABFT ablations:
# full ABFT, partials only (no checksum rows, no checks), and everything off but the flag.
mkdir -p gpurun_out
for m in 0 23 31; do
  ABFT_DEV_ABLATE=$m timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_update_ws -s 1 -c 1 \
     -o gpurun_out/upd_ablate$m -f python tools/run_once.py 32768 512 > gpurun_out/ncu_upd_ablate$m.log 2>&1
done
