mkdir -p gpurun_out
for g in 1 2 4 10 16; do
  ABFT_CHOL_G=$g timeout 300 python tools/c2_ablate.py 4096 256 | sed "s/^{/{\"G\": $g, /" >> gpurun_out/chol_g.jsonl
  ABFT_CHOL_G=$g timeout 300 python tools/c2_ablate.py 16384 512 | sed "s/^{/{\"G\": $g, /" >> gpurun_out/chol_g.jsonl
done
ABFT_CHOL=recursive timeout 300 python tools/c2_ablate.py 4096 256 | sed 's/^{/{"G": "recursive", /' >> gpurun_out/chol_g.jsonl
