set -x
timeout 1500 python tools/ab.py "base|" "wf||MSCCL_LIB=/root/repo/tools/variants/lib_wf.so" "rs||MSCCL_LIB=/root/repo/tools/variants/lib_rs.so" "ag|--program allgather" "ag_wf|--program allgather|MSCCL_LIB=/root/repo/tools/variants/lib_wf.so" "rsc|--program reducescatter" "rsc_wf|--program reducescatter|MSCCL_LIB=/root/repo/tools/variants/lib_wf.so" --reps 3 > gpurun_out/ab_r2d.log 2>&1; grep SUMMARY gpurun_out/ab_r2d.log
mkdir -p gpurun_out/ncu
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mscclInterpreter -c 1 -s 3 -o gpurun_out/ncu/rs_r2 python bench.py --program reducescatter --steps 1 --warmup 3 --no-cpu --no-e2e --quiet-extra > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mscclInterpreter -c 1 -s 3 -o gpurun_out/ncu/ag_r2 python bench.py --program allgather --steps 1 --warmup 3 --no-cpu --no-e2e --quiet-extra > /dev/null 2>&1
ls -la gpurun_out/ncu
