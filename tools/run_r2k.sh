python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 2400 python -m pytest tests -m gpu -q -rs > gpurun_out/gputest_r2k.log 2>&1; tail -4 gpurun_out/gputest_r2k.log
/usr/bin/time -f "bench wall %e s" timeout 900 python bench.py > gpurun_out/bench_r2k.json 2> gpurun_out/bench_r2k.err; tail -1 gpurun_out/bench_r2k.err; python -c "import json;d=json.load(open('gpurun_out/bench_r2k.json'));print(d['value'], d['roofline']['frac'], json.dumps(d['extras']['allreduce_1KiB_fp16_latency_us']))"
MSCCL_FORCE_DEVICE=0 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 --size-mib 1 > gpurun_out/bench_tr2k.json 2> gpurun_out/bench_tr2k.err; tail -c 1200 gpurun_out/bench_tr2k.json
timeout 1200 python bench.py --sweep gpurun_out/sweep_r2k.jsonl > gpurun_out/sweep_r2k.log 2>&1; wc -l gpurun_out/sweep_r2k.jsonl
