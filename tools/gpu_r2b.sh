free -g | head -2
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_r2b.log; tail -5 gpurun_out/pytest_r2b.log
timeout 600 python bench.py > gpurun_out/bench_r2b.json 2> gpurun_out/bench_r2b.err; tail -3 gpurun_out/bench_r2b.err; head -c 600 gpurun_out/bench_r2b.json
CUSZP_BENCH_SHARE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 3 --warmup 3 > gpurun_out/bench_r2b_share2.json 2> gpurun_out/bench_r2b_share2.err; tail -3 gpurun_out/bench_r2b_share2.err; head -c 400 gpurun_out/bench_r2b_share2.json
timeout 600 python bench.py --impl reference > gpurun_out/bench_r2b_ref.json 2> gpurun_out/bench_r2b_ref.err; tail -2 gpurun_out/bench_r2b_ref.err; cat gpurun_out/bench_r2b_ref.json
