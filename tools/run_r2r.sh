python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 2400 python -m pytest tests -m gpu -q -rs > gpurun_out/gputest_r2r.log 2>&1; tail -3 gpurun_out/gputest_r2r.log
timeout 900 python bench.py > gpurun_out/bench_r2r.json 2> gpurun_out/bench_r2r.err; python -c "import json;d=json.load(open('gpurun_out/bench_r2r.json'));print(d['value'], d['roofline']['frac'], d['e2e']['value'], d['e2e']['serial_ms_per_step'], d['cpu_baseline']['value'])"
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 | tail -c 400
