O=gpurun_out/r01d; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_exchange.py -q -x 2>&1 | tail -15
PSB_DIST_BACKEND=gloo PSB_BENCH_DEVICE=0 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --mode data --config C2 --steps 20 --warmup 3 --no-extras > $O/bench_data2_p2p_1gpu.json 2> $O/bench_data2_p2p_1gpu.err
tail -3 $O/bench_data2_p2p_1gpu.err; cat $O/bench_data2_p2p_1gpu.json | head -c 1500
