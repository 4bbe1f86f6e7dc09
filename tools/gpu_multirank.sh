cd $GRAFT_REPO_ROOT
IPT_BENCH_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 3 --warmup 3 --no-e2e --no-cpu --workload c5 > gpurun_out/bench_mr_c5.json 2> gpurun_out/bench_mr.err
IPT_BENCH_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu --e2e-steps 1 > gpurun_out/bench_mr_sweep.json 2>> gpurun_out/bench_mr.err
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29535 bench.py --impl reference --gpus 2 --steps 1 --warmup 1 > gpurun_out/bench_mr_ref.json 2>> gpurun_out/bench_mr.err
