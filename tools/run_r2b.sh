set -x
python -m pytest tests/test_gpu_multiprocess.py -x -q > gpurun_out/mp_r2b.log 2>&1; tail -3 gpurun_out/mp_r2b.log
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_r2b.json 2> gpurun_out/bench_r2b.err; tail -c 1500 gpurun_out/bench_r2b.json; tail -5 gpurun_out/bench_r2b.err
MSCCL_FORCE_DEVICE=0 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 5 --warmup 3 --size-mib 2 > gpurun_out/bench_tr2.json 2> gpurun_out/bench_tr2.err; tail -c 3000 gpurun_out/bench_tr2.json; tail -5 gpurun_out/bench_tr2.err
timeout 900 python bench.py --sweep gpurun_out/sweep_r2.jsonl > gpurun_out/sweep_r2.log 2>&1; tail -3 gpurun_out/sweep_r2.log
