timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/gputest_r2g.log 2>&1; tail -3 gpurun_out/gputest_r2g.log
timeout 600 python bench.py > gpurun_out/bench_r2g.json 2> gpurun_out/bench_r2g.err; python -c "import json;d=json.load(open('gpurun_out/bench_r2g.json'));print(d['value'], d['roofline']['frac'], json.dumps(d['extras']))"
timeout 600 python bench.py --program nvls --no-cpu --no-e2e --quiet-extra --steps 10 > gpurun_out/bench_nvls_r2g.json 2>&1; tail -c 600 gpurun_out/bench_nvls_r2g.json
