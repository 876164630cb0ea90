# Code-path check of bench.py at N > 1 on ONE GPU (not a measurement: the ranks share the device):
# two ranks, peer-memory transport, 1D and 2D (2 x 1) layouts.
mkdir -p gpurun_out
for pr in 1 2; do
  BENCH_SHARE_DEVICE=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
      --master-port $((29500 + pr)) bench.py --gpus 2 --steps 2 --warmup 3 --matrix-n 8192 --nb 512 --prows $pr \
      > gpurun_out/bench_mr_p$pr.log 2> gpurun_out/bench_mr_p$pr.err; echo rc=$? >> gpurun_out/bench_mr_p$pr.err
done
