# Round-2 final pass after the streamed host input: GPU suite, bench line, smoke
mkdir -p gpurun_out
( time timeout 1500 python -m pytest tests -m gpu -q ) > gpurun_out/final2_gputests.log 2>&1; echo rc=$? >> gpurun_out/final2_gputests.log
( time timeout 900 python bench.py ) > gpurun_out/final2_bench.log 2> gpurun_out/final2_bench.err; echo rc=$? >> gpurun_out/final2_bench.err
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final2_smoke.log 2>&1; echo rc=$? >> gpurun_out/final2_smoke.log
