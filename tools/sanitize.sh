# compute-sanitizer over the torch-free driver (tools/sanitize_driver.cu), small size.
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  ABFT_GRAPH=0 timeout 900 compute-sanitizer --tool $tool --print-limit 50 tools/bin/sanitize_driver ${N:-1024} ${NB:-256} > gpurun_out/sanitize_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/sanitize_$tool.log
done
