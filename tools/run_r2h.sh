timeout 1200 python -m pytest tests/test_gpu_nvls.py -x -q > gpurun_out/nvls_r2h.log 2>&1; tail -2 gpurun_out/nvls_r2h.log
timeout 600 python bench.py > gpurun_out/bench_r2h.json 2> gpurun_out/bench_r2h.err; python -c "import json;d=json.load(open('gpurun_out/bench_r2h.json'));print(d['value'], d['roofline']['frac'], json.dumps(d['extras']))"
mkdir -p gpurun_out/ncu
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/ncu/launches_r2h.csv python bench.py --steps 2 --warmup 1 --no-cpu --no-e2e > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mscclInterpreter -c 1 -s 3 -o gpurun_out/ncu/ring_r2h python bench.py --steps 1 --warmup 3 --no-cpu --no-e2e --quiet-extra > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mscclInterpreter -c 1 -s 3 -o gpurun_out/ncu/nvls_r2h python bench.py --program nvls --steps 1 --warmup 3 --no-cpu --no-e2e --quiet-extra > /dev/null 2>&1
ls -la gpurun_out/ncu
