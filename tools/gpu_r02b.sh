# Re-validation of HEAD after the stage-release fix: GPU suite, bench line, reference arm, smoke, launch list.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt
( time timeout 1500 python -m pytest tests -m gpu -x -q ) > gpurun_out/gputests.log 2>&1; echo rc=$? >> gpurun_out/gputests.log
( time timeout 900 python bench.py ) > gpurun_out/bench.log 2> gpurun_out/bench.err; echo rc=$? >> gpurun_out/bench.err
( time timeout 600 python bench.py --impl reference --steps 2 --warmup 3 ) > gpurun_out/bench_ref.log 2>&1; echo rc=$? >> gpurun_out/bench_ref.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo rc=$? >> gpurun_out/smoke.log
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/launches_c4.csv \
    python bench.py --no-extras --steps 1 --warmup 0 > gpurun_out/ncu_launch_run.log 2>&1; echo rc=$? >> gpurun_out/ncu_launch_run.log
