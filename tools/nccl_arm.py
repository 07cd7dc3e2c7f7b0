"""NCCL comparison arm for bench.py (SURVEY §8(d) "NCCL baseline"): NCCL 2.28.9 called
through ctypes on the torch-bundled libnccl.so.2, in the same process model and timing loop
as the MSCCL interpreter. It is a BASELINE only -- nothing on the measured MSCCL path calls
NCCL. One communicator per process (one rank per GPU); NCCL refuses two ranks on one GPU,
so on a single-GPU box the arm is skipped with that reason.
"""
import ctypes
import glob
import os

_DT = {"int8": 0, "uint8": 1, "int32": 2, "uint32": 3, "int64": 4, "uint64": 5, "float16": 6, "float32": 7,
       "float64": 8, "bfloat16": 9}
_OP = {"sum": 0, "prod": 1, "max": 2, "min": 3}


def _libpath():
    import torch
    base = os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "nccl", "lib")
    c = sorted(glob.glob(os.path.join(base, "libnccl.so*")))
    return c[0] if c else "libnccl.so.2"


class NcclUniqueId(ctypes.Structure):
    _fields_ = [("internal", ctypes.c_byte * 128)]


class Nccl:
    def __init__(self):
        self.lib = ctypes.CDLL(_libpath())
        v = ctypes.c_int()
        self.lib.ncclGetVersion(ctypes.byref(v))
        self.version = v.value
        vp, sz, i = ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int
        self.lib.ncclAllReduce.argtypes = [vp, vp, sz, i, i, vp, vp]
        self.lib.ncclAlltoAll.argtypes = [vp, vp, sz, i, vp, vp]
        self.lib.ncclAllGather.argtypes = [vp, vp, sz, i, vp, vp]
        self.lib.ncclReduceScatter.argtypes = [vp, vp, sz, i, i, vp, vp]
        self.lib.ncclCommInitRank.argtypes = [ctypes.POINTER(vp), i, NcclUniqueId, i]
        self.lib.ncclCommDestroy.argtypes = [vp]
        self.lib.ncclGetErrorString.restype = ctypes.c_char_p
        self.comm = None

    def _chk(self, r):
        if r != 0:
            raise RuntimeError("nccl error %d: %s" % (r, self.lib.ncclGetErrorString(r).decode()))

    def init(self, rank, world):
        """Rank 0 creates the unique id; it travels over torch.distributed (plumbing only)."""
        import torch.distributed as dist
        uid = NcclUniqueId()
        if rank == 0:
            self._chk(self.lib.ncclGetUniqueId(ctypes.byref(uid)))
        obj = [bytes(uid.internal) if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        ctypes.memmove(uid.internal, obj[0], 128)
        c = ctypes.c_void_p()
        self._chk(self.lib.ncclCommInitRank(ctypes.byref(c), world, uid, rank))
        self.comm = c
        return self

    def allreduce(self, x, y, dtype, op="sum", stream=0):
        self._chk(self.lib.ncclAllReduce(x.data_ptr(), y.data_ptr(), x.numel(), _DT[dtype], _OP[op], self.comm,
                                         stream))

    def alltoall(self, x, y, dtype, world, stream=0):
        self._chk(self.lib.ncclAlltoAll(x.data_ptr(), y.data_ptr(), x.numel() // world, _DT[dtype], self.comm, stream))

    def allgather(self, x, y, dtype, stream=0):
        self._chk(self.lib.ncclAllGather(x.data_ptr(), y.data_ptr(), x.numel(), _DT[dtype], self.comm, stream))

    def reducescatter(self, x, y, dtype, op="sum", stream=0):
        self._chk(self.lib.ncclReduceScatter(x.data_ptr(), y.data_ptr(), y.numel(), _DT[dtype], _OP[op], self.comm,
                                             stream))

    def destroy(self):
        if self.comm:
            self.lib.ncclCommDestroy(self.comm)
            self.comm = None
