# Round-end style GPU run: bench line (timed), reference arm, smoke, ncu launch list of one step.
mkdir -p gpurun_out
( time timeout 1200 python bench.py ) > gpurun_out/bench.log 2> gpurun_out/bench.err; echo rc=$? >> gpurun_out/bench.err
( time timeout 900 python bench.py --impl reference ) > gpurun_out/bench_ref.log 2> gpurun_out/bench_ref.err; echo rc=$? >> gpurun_out/bench_ref.err
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo rc=$? >> gpurun_out/smoke.log
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 3600 --csv --log-file gpurun_out/launches_c4.csv \
    python bench.py --no-extras --steps 1 --warmup 0 > gpurun_out/ncu_launch_run.log 2>&1; echo rc=$? >> gpurun_out/ncu_launch_run.log
