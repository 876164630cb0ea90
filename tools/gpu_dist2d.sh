mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_dist2d.py -x -q > gpurun_out/dist2d.log 2>&1; echo rc=$? >> gpurun_out/dist2d.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/gputests2.log 2>&1; echo rc=$? >> gpurun_out/gputests2.log
