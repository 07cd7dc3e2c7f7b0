for lib in "" tools/variants/*.so; do echo "== ${lib:-default}"; MSCCL_LIB=$lib timeout 300 python tools/tune8.py 2>&1 | grep -v error | tail -10; done
