"""ctypes binding to libmsccl_b200.so — argument marshalling only.

Every function here forwards to the C ABI of ``include/msccl.h`` with the same name
(minus the ``mscclXxx`` prefix); all data movement and reduction happens in the CUDA
interpreter kernel. If the shared library is missing this module raises at import:
there is no CPU fallback.

torch is used for device memory and streams only (tensors are passed by data pointer).
"""
import contextlib
import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIBPATH = os.environ.get("MSCCL_LIB") or os.path.join(_HERE, "libmsccl_b200.so")

if not os.path.exists(LIBPATH):
    raise ImportError("libmsccl_b200.so not built (run `make` or __graft_entry__.build()); "
                      "the MSCCL interpreter has no fallback")
lib = ctypes.CDLL(LIBPATH)

HANDLE_BYTES = 128
REG_DESC_BYTES = 128
RESULTS = {0: "Success", 1: "UnhandledCudaError", 2: "SystemError", 3: "InternalError", 4: "InvalidArgument",
           5: "InvalidUsage", 6: "RemoteError", 7: "InProgress", 8: "InvalidProgram", 9: "NoMatchingProgram"}
DTYPES = {"int8": 0, "uint8": 1, "int32": 2, "uint32": 3, "int64": 4, "uint64": 5, "float16": 6, "float32": 7,
          "float64": 8, "bfloat16": 9}
OPS = {"sum": 0, "prod": 1, "max": 2, "min": 3}

_c = ctypes
_vp, _sz, _i, _i64 = _c.c_void_p, _c.c_size_t, _c.c_int, _c.c_int64
SIGNATURES = {
    "mscclCommInitAll": (_i, [_c.POINTER(_vp), _i, _c.POINTER(_i)]),
    "mscclCommInitRank": (_i, [_c.POINTER(_vp), _i, _i, _i]),
    "mscclCommExportHandle": (_i, [_vp, _vp, _c.POINTER(_sz)]),
    "mscclCommConnect": (_i, [_vp, _vp]),
    "mscclCommDestroy": (_i, [_vp]),
    "mscclCommCount": (_i, [_vp, _c.POINTER(_i)]),
    "mscclCommUserRank": (_i, [_vp, _c.POINTER(_i)]),
    "mscclCommCuDevice": (_i, [_vp, _c.POINTER(_i)]),
    "mscclCommGetAsyncError": (_i, [_vp, _c.POINTER(_i)]),
    "mscclLoadProgram": (_i, [_vp, _c.c_char_p, _sz, _sz, _sz, _c.POINTER(_vp)]),
    "mscclUnloadProgram": (_i, [_vp, _vp]),
    "mscclProgramInfo": (_i, [_vp, _c.POINTER(_i), _c.POINTER(_i), _c.POINTER(_i)]),
    "mscclValidateProgram": (_i, [_c.c_char_p, _sz, _i, _i, _i, _c.c_char_p, _sz]),
    "mscclProgramTouches": (_i, [_vp, _i, _c.POINTER(_i64)]),
    "mscclAllReduce": (_i, [_vp, _vp, _sz, _i, _i, _vp, _vp]),
    "mscclAllGather": (_i, [_vp, _vp, _sz, _i, _vp, _vp]),
    "mscclReduceScatter": (_i, [_vp, _vp, _sz, _i, _i, _vp, _vp]),
    "mscclAllToAll": (_i, [_vp, _vp, _sz, _i, _vp, _vp]),
    "mscclRunProgram": (_i, [_vp, _vp, _vp, _sz, _i, _i, _vp, _vp]),
    "mscclGroupStart": (_i, []),
    "mscclGroupEnd": (_i, []),
    "mscclGetErrorString": (_c.c_char_p, [_i]),
    "mscclGetLastError": (_c.c_char_p, [_vp]),
    "mscclSetParam": (_i, [_c.c_char_p, _i64]),
    "mscclGetParam": (_i, [_c.c_char_p, _c.POINTER(_i64)]),
    "mscclLaunchCount": (_c.c_uint64, []),
    "mscclCommGetStats": (_i, [_vp, _c.POINTER(_i64), _i]),
    "mscclCommRegister": (_i, [_vp, _vp, _sz, _c.POINTER(_vp)]),
    "mscclNvlsSupported": (_i, [_i, _c.POINTER(_i)]),
    "mscclNvlsAlloc": (_i, [_c.POINTER(_vp), _i, _sz, _c.POINTER(_vp)]),
    "mscclNvlsFree": (_i, [_c.POINTER(_vp), _i, _c.POINTER(_vp)]),
    "mscclRegExport": (_i, [_vp, _vp]),
    "mscclRegConnect": (_i, [_vp, _vp]),
    "mscclCommDeregister": (_i, [_vp, _vp]),
    "mscclDebugSetGeneration": (_i, [_vp, _c.c_uint64]),
    "mscclDebugDirectPlacement": (_i, [_c.c_char_p, _sz, _i, _c.POINTER(_c.c_int32), _c.POINTER(_c.c_int32), _i,
                                       _c.POINTER(_i)]),
}
for _name, (_res, _args) in SIGNATURES.items():
    _f = getattr(lib, _name)
    _f.restype = _res
    _f.argtypes = _args
_run_program = lib.mscclRunProgram


class MscclError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__("msccl %s (%d): %s" % (RESULTS.get(code, "?"), code, msg))
        self.code = code


def _check(code, comm=None):
    if code != 0:
        raise MscclError(code, lib.mscclGetLastError(comm).decode(errors="replace"))


def set_param(key, value):
    _check(lib.mscclSetParam(key.encode(), int(value)))


def get_param(key):
    v = _i64()
    _check(lib.mscclGetParam(key.encode(), _c.byref(v)))
    return v.value


def launch_count():
    return int(lib.mscclLaunchCount())


def validate(ir_text, nranks, slots=0, max_tbs=0):
    """C++ validator (rules V1..V9) without a GPU. Returns (ok, message)."""
    b = ir_text.encode() if isinstance(ir_text, str) else ir_text
    err = _c.create_string_buffer(1024)
    r = lib.mscclValidateProgram(b, len(b), nranks, slots, max_tbs, err, 1024)
    return r == 0, err.value.decode()


def direct_placement(ir_text, rank):
    """The loader's direct-placement marking for `rank` (mscclDebugDirectPlacement, no GPU):
    a list, in (thread block, step) order, of (flags, rdst_buf, rdst_chunk) with flags bit 0 =
    direct send, bit 1 = direct receive (reading R15), bit 2 = pulled receive, bit 3 = pulled send
    (reading R30)."""
    b = ir_text.encode() if isinstance(ir_text, str) else ir_text
    n = _i()
    _check(lib.mscclDebugDirectPlacement(b, len(b), rank, None, None, 0, _c.byref(n)))
    flags = (_c.c_int32 * max(1, n.value))()
    rdst = (_c.c_int32 * max(2, 2 * n.value))()
    _check(lib.mscclDebugDirectPlacement(b, len(b), rank, flags, rdst, n.value, _c.byref(n)))
    return [(flags[k], rdst[2 * k], rdst[2 * k + 1]) for k in range(n.value)]


def nvls_supported(device):
    """mscclNvlsSupported: NVSwitch multicast support of a device (bool)."""
    v = _i()
    _check(lib.mscclNvlsSupported(device, _c.byref(v)))
    return bool(v.value)


class _DeviceMemory:
    """A raw device range exposed through __cuda_array_interface__ (zero-copy torch view)."""

    def __init__(self, ptr, nbytes):
        self.__cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (ptr, False),
                                         "version": 3, "strides": None}


def nvls_alloc(comms, nbytes):
    """mscclNvlsAlloc over a full rank-ordered communicator set: one uint8 torch tensor per
    rank (views of the multicast-bound memory; free with nvls_free)."""
    import torch
    n = len(comms)
    arr = (_vp * n)(*[c.handle for c in comms])
    ptrs = (_vp * n)()
    _check(lib.mscclNvlsAlloc(arr, n, nbytes, ptrs), comms[0].handle)
    out = []
    for i, c in enumerate(comms):
        with torch.cuda.device(_device_of(c)):
            out.append(torch.as_tensor(_DeviceMemory(ptrs[i], nbytes), device="cuda"))
    return out, [ptrs[i] for i in range(n)]


def nvls_free(comms, ptrs):
    n = len(comms)
    arr = (_vp * n)(*[c.handle for c in comms])
    p = (_vp * n)(*ptrs)
    _check(lib.mscclNvlsFree(arr, n, p), comms[0].handle)


def _device_of(comm):
    v = _i()
    _check(lib.mscclCommCuDevice(comm.handle, _c.byref(v)))
    return v.value


_TORCH_DT = None


def _dtype_name(t):
    global _TORCH_DT
    if _TORCH_DT is None:  # built once: this sits on the per-call path
        import torch
        m = {torch.int8: "int8", torch.uint8: "uint8", torch.int32: "int32", torch.int64: "int64",
             torch.float16: "float16", torch.float32: "float32", torch.float64: "float64",
             torch.bfloat16: "bfloat16"}
        for k in ("uint32", "uint64"):
            if hasattr(torch, k):
                m[getattr(torch, k)] = k
        _TORCH_DT = m
    return _TORCH_DT[t.dtype]


_RAW_STREAM = None


def _stream(stream, device=None):
    """cudaStream_t of `stream`, or of the current stream of `device` (the per-call path:
    torch's raw-stream query avoids building a Stream object on every call)."""
    global _RAW_STREAM
    if stream is None:
        if _RAW_STREAM is None:
            import torch
            _RAW_STREAM = getattr(torch._C, "_cuda_getCurrentRawStream", None) or \
                (lambda d: torch.cuda.current_stream(d).cuda_stream)
        if device is None:
            import torch
            device = torch.cuda.current_device()
        return _RAW_STREAM(device)
    s = getattr(stream, "cuda_stream", None)
    return s if s is not None else int(stream)


@contextlib.contextmanager
def group():
    """mscclGroupStart / mscclGroupEnd (one cooperative launch per device at exit)."""
    _check(lib.mscclGroupStart())
    ok = False
    try:
        yield
        ok = True
    finally:
        r = lib.mscclGroupEnd()
        if ok:
            _check(r)


class Program:
    def __init__(self, comm, handle):
        self.comm = comm
        self.handle = handle

    def info(self):
        a, b, c = _i(), _i(), _i()
        _check(lib.mscclProgramInfo(self.handle, _c.byref(a), _c.byref(b), _c.byref(c)), self.comm.handle)
        return {"thread_blocks": a.value, "instructions": b.value, "inplace": bool(c.value)}

    def set_generation(self, gen):
        """mscclDebugSetGeneration (test hook): the launch generation of every thread block."""
        _check(lib.mscclDebugSetGeneration(self.handle, gen), self.comm.handle)

    def touches(self, direct=True):
        """Algorithmic chunk-sized memory touches of this rank's program (mscclProgramTouches)."""
        v = _i64()
        _check(lib.mscclProgramTouches(self.handle, int(direct), _c.byref(v)), self.comm.handle)
        return v.value


class Registration:
    """A registered buffer (mscclReg_t)."""

    def __init__(self, comm, handle):
        self.comm = comm
        self.handle = handle

    def export(self):
        buf = _c.create_string_buffer(REG_DESC_BYTES)
        _check(lib.mscclRegExport(self.handle, buf), self.comm.handle)
        return buf.raw

    def connect(self, all_descs):
        _check(lib.mscclRegConnect(self.handle, b"".join(all_descs)), self.comm.handle)

    def deregister(self):
        if self.handle:
            _check(lib.mscclCommDeregister(self.comm.handle, self.handle), self.comm.handle)
            self.handle = None


class Comm:
    """One rank (mscclComm_t)."""

    def __init__(self, handle):
        self.handle = _vp(handle) if not isinstance(handle, _vp) else handle
        self.programs = []
        d = _i()
        _check(lib.mscclCommCuDevice(self.handle, _c.byref(d)))
        self.device = d.value

    # --- construction
    @staticmethod
    def init_all(devices):
        """mscclCommInitAll; repeated device ids are virtual ranks on one GPU."""
        n = len(devices)
        arr = (_vp * n)()
        dl = (_i * n)(*devices)
        _check(lib.mscclCommInitAll(arr, n, dl))
        return [Comm(arr[i]) for i in range(n)]

    @staticmethod
    def virtual(nranks, device=0):
        return Comm.init_all([device] * nranks)

    @staticmethod
    def init_rank(nranks, rank, device):
        h = _vp()
        _check(lib.mscclCommInitRank(_c.byref(h), nranks, rank, device))
        return Comm(h)

    def export_handle(self):
        buf = _c.create_string_buffer(HANDLE_BYTES)
        _check(lib.mscclCommExportHandle(self.handle, buf, None), self.handle)
        return buf.raw

    def connect(self, all_handles):
        blob = b"".join(all_handles)
        _check(lib.mscclCommConnect(self.handle, blob), self.handle)

    def destroy(self):
        if self.handle:
            _check(lib.mscclCommDestroy(self.handle))
            self.handle = None

    # --- attributes
    @property
    def rank(self):
        v = _i()
        _check(lib.mscclCommUserRank(self.handle, _c.byref(v)))
        return v.value

    @property
    def nranks(self):
        v = _i()
        _check(lib.mscclCommCount(self.handle, _c.byref(v)))
        return v.value

    def async_error(self):
        v = _i()
        _check(lib.mscclCommGetAsyncError(self.handle, _c.byref(v)))
        return v.value

    def stats(self):
        """mscclCommGetStats: {"cross_direct_handshakes", "launches_direct1", "launches_direct2",
        "multicast_pieces", "depth_checks"}."""
        v = (_i64 * 5)()
        _check(lib.mscclCommGetStats(self.handle, v, 5), self.handle)
        return {"cross_direct_handshakes": v[0], "launches_direct1": v[1], "launches_direct2": v[2],
                "multicast_pieces": v[3], "depth_checks": v[4]}

    def last_error(self):
        return lib.mscclGetLastError(self.handle).decode(errors="replace")

    # --- buffer registration (direct placement across processes, reading R15b)
    def register(self, tensor_or_ptr, nbytes=None):
        """mscclCommRegister: returns a Registration; export()/connect() complete it."""
        if nbytes is None:
            ptr, nbytes = tensor_or_ptr.data_ptr(), tensor_or_ptr.numel() * tensor_or_ptr.element_size()
        else:
            ptr = int(tensor_or_ptr)
        h = _vp()
        _check(lib.mscclCommRegister(self.handle, _vp(ptr), nbytes, _c.byref(h)), self.handle)
        return Registration(self, h)

    # --- programs
    def load(self, ir_text, min_bytes=0, max_bytes=0):
        b = ir_text.encode() if isinstance(ir_text, str) else ir_text
        h = _vp()
        _check(lib.mscclLoadProgram(self.handle, b, len(b), min_bytes, max_bytes, _c.byref(h)), self.handle)
        p = Program(self, h)
        self.programs.append(p)
        return p

    def unload(self, prog):
        _check(lib.mscclUnloadProgram(self.handle, prog.handle), self.handle)
        self.programs.remove(prog)

    # --- collectives (torch tensors; counts in elements)
    def allreduce(self, send, recv, op="sum", stream=None, count=None):
        n = send.numel() if count is None else count
        _check(lib.mscclAllReduce(_vp(send.data_ptr()), _vp(recv.data_ptr()), n, DTYPES[_dtype_name(send)],
                                  OPS[op], self.handle, _stream(stream, self.device)), self.handle)

    def allgather(self, send, recv, stream=None):
        _check(lib.mscclAllGather(_vp(send.data_ptr()), _vp(recv.data_ptr()), send.numel(),
                                  DTYPES[_dtype_name(send)], self.handle, _stream(stream, self.device)), self.handle)

    def reducescatter(self, send, recv, op="sum", stream=None):
        _check(lib.mscclReduceScatter(_vp(send.data_ptr()), _vp(recv.data_ptr()), recv.numel(),
                                      DTYPES[_dtype_name(send)], OPS[op], self.handle, _stream(stream, self.device)), self.handle)

    def alltoall(self, send, recv, stream=None):
        n = send.numel() // self.nranks
        _check(lib.mscclAllToAll(_vp(send.data_ptr()), _vp(recv.data_ptr()), n, DTYPES[_dtype_name(send)],
                                 self.handle, _stream(stream, self.device)), self.handle)

    def run(self, prog, send, recv, count, op="sum", stream=None, dtype=None):
        dt = DTYPES[dtype or _dtype_name(send)]
        r = _run_program(prog.handle, send.data_ptr(), recv.data_ptr(), count, dt, OPS[op], self.handle,
                         _stream(stream, self.device))
        if r:
            _check(r, self.handle)
