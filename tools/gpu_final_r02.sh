# End-of-round evidence at HEAD (round 2): GPU suite, bench line, reference arm, smoke, ncu launch
# list of one C4 step, ncu --set full of the dominant kernel (update (b) of iteration 0 at C4, the
# second k_update_ws launch), compute-sanitizer over the torch-free driver (incl. 1D/2D dist harness).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv > gpurun_out/final_gpu.txt
( time timeout 1500 python -m pytest tests -m gpu -q ) > gpurun_out/final_gputests.log 2>&1; echo rc=$? >> gpurun_out/final_gputests.log
( time timeout 900 python bench.py ) > gpurun_out/final_bench.log 2> gpurun_out/final_bench.err; echo rc=$? >> gpurun_out/final_bench.err
( time timeout 600 python bench.py --impl reference --steps 2 --warmup 3 ) > gpurun_out/final_bench_ref.log 2>&1; echo rc=$? >> gpurun_out/final_bench_ref.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_smoke.log 2>&1; echo rc=$? >> gpurun_out/final_smoke.log
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/final_launches_c4.csv \
    python bench.py --no-extras --steps 1 --warmup 0 > gpurun_out/final_ncu_launch.log 2>&1; echo rc=$? >> gpurun_out/final_ncu_launch.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_update_ws -s 1 -c 1 \
    -o gpurun_out/final_update_full -f python tools/run_once.py 32768 512 > gpurun_out/final_ncu_full.log 2>&1; echo rc=$? >> gpurun_out/final_ncu_full.log
bash tools/sanitize.sh
