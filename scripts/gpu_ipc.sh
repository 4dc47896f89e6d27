# IPC backend: 2-process parity tests on one GPU, then a 2-rank bench (both ranks on GPU 0)
timeout -s KILL 900 python -m pytest tests/test_gpu_ipc.py -q --timeout 300 -x 2>&1 | tail -15
timeout -s KILL 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
   --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --comm ipc --no-e2e --no-cpu-baseline --no-cache-l0 \
   > gpurun_out/bench_ipc2.json 2> gpurun_out/bench_ipc2.err; echo "bench ipc rc=$?"
tail -5 gpurun_out/bench_ipc2.err; cat gpurun_out/bench_ipc2.json
timeout -s KILL 1200 python -m pytest tests -m gpu -q --timeout 300 -x 2>&1 | tail -5
