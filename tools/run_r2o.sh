timeout 2400 python -m pytest tests -m gpu -q -rs > gpurun_out/gputest_r2o.log 2>&1; tail -3 gpurun_out/gputest_r2o.log
timeout 900 python bench.py > gpurun_out/bench_r2o.json 2> gpurun_out/bench_r2o.err; python -c "import json;d=json.load(open('gpurun_out/bench_r2o.json'));print(d['value'], d['roofline']['frac'], d['e2e'], json.dumps(d['extras']))"
timeout 900 python tools/ab.py "nvls32|--program nvls --instances 32" "nvls36|--program nvls --instances 36" --reps 1 > gpurun_out/ab_r2o.log 2>&1; grep SUMMARY gpurun_out/ab_r2o.log
