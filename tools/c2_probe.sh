# Small-n critical path probe (C2 >= 8 TFLOP/s): interleaved ABFT on/off with the
# phase breakdown at C2 and C3, and an ncu launch list of one C2 factorisation.
mkdir -p gpurun_out
for cfg in "4096 256" "16384 512"; do
  timeout 600 python tools/time_arms.py $cfg 5 >> gpurun_out/arms_small.jsonl 2>> gpurun_out/arms_small.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches_c2.csv \
    python bench.py --n 4096 --nb 256 --no-extras --steps 1 --warmup 0 > gpurun_out/ncu_c2.log 2>&1; echo rc=$? >> gpurun_out/ncu_c2.log
