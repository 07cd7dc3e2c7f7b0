V=/root/repo/tools/variants/lib_dyn.so
MSCCL_LIB=$V timeout 600 python -m pytest tests/test_gpu_large.py tests/test_gpu_parity.py -x -q > gpurun_out/dyn_tests.log 2>&1; tail -2 gpurun_out/dyn_tests.log
timeout 1500 python tools/ab.py "base|" "dyn||MSCCL_LIB=$V" "rs|--program reducescatter" "rs_dyn|--program reducescatter|MSCCL_LIB=$V" "ag|--program allgather" "ag_dyn|--program allgather|MSCCL_LIB=$V" "a2a|--program alltoall --instances 2" "a2a_dyn|--program alltoall --instances 2|MSCCL_LIB=$V" --reps 3 > gpurun_out/ab_r2m.log 2>&1; grep SUMMARY gpurun_out/ab_r2m.log
