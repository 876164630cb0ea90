# compute-sanitizer over the torch-free driver (tools/sanitize_driver.cu), small size: the update GEMM,
# single-GPU factorisations, and the multi-GPU driver (1D and 2D block-cyclic) in the one-device harness.
mkdir -p gpurun_out tools/bin
nvcc -std=c++17 -O2 -o tools/bin/sanitize_driver tools/sanitize_driver.cu -Lpaper_conf_ipps_chenlc16_b200 -l:libabft.so \
     -Xlinker -rpath=$PWD/paper_conf_ipps_chenlc16_b200
for tool in memcheck racecheck synccheck initcheck; do
  ABFT_GRAPH=0 timeout 900 compute-sanitizer --tool $tool --print-limit 50 tools/bin/sanitize_driver ${N:-1024} ${NB:-256} > gpurun_out/sanitize_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/sanitize_$tool.log
done
