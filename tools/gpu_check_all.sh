# GPU suite + default bench line + small-n arms (after a driver change)
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/gputests.log 2>&1; echo rc=$? >> gpurun_out/gputests.log
timeout 900 python bench.py > gpurun_out/bench.log 2> gpurun_out/bench.err; echo rc=$? >> gpurun_out/bench.err
for cfg in "4096 256" "16384 512"; do
  timeout 600 python tools/time_arms.py $cfg 5 >> gpurun_out/arms_small.jsonl 2>> gpurun_out/arms_small.err
done
