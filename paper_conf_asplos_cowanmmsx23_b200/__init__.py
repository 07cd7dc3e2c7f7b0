"""B200-native MSCCL-IR interpreter (MSCCLang, ASPLOS '23 — data-parallel hot path).

* ``dsl`` / ``programs`` — the chunk-oriented DSL and its lowering to MSCCL-IR.
* ``ir``                 — the IR model and its text form.
* ``runtime``            — ctypes binding to ``libmsccl_b200.so`` (the C ABI declared in
                           ``include/msccl.h``); every collective runs in the CUDA
                           interpreter kernel. There is no CPU fallback.
"""
from . import ir, dsl, programs  # noqa: F401
