# C2 / C3 critical-path attribution: tools/c2_ablate.py per ABFT_DEV_ABLATE mask (one process each)
mkdir -p gpurun_out
for cfg in "4096 256" "16384 512"; do
  for m in 0 1 2 4 8 16 31; do
    ABFT_DEV_ABLATE=$m timeout 300 python tools/c2_ablate.py $cfg >> gpurun_out/c2_ablate.jsonl 2>> gpurun_out/c2_ablate.err
  done
done
