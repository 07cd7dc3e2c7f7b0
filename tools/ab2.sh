for lib in "" tools/variants/*.so; do MSCCL_LIB=$lib timeout 300 python tools/tune7.py 2>&1 | grep -v "^$" | tail -6; done
