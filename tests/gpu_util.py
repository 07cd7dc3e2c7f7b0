"""Helpers for the -m gpu tests: run IR programs through the C ABI on virtual ranks."""
import numpy as np
import torch

from paper_conf_asplos_cowanmmsx23_b200 import runtime

_COMMS = {}


def comms(R, device=0):
    """Cached virtual-rank communicator set (one region allocation per R and parameter set)."""
    key = (R, device) + tuple(runtime.get_param(k) for k in ("MSCCL_SLOTS", "MSCCL_SLOT_BYTES", "MSCCL_THREADS",
                                                              "MSCCL_MAX_CHANNELS", "MSCCL_TIMEOUT_S",
                                                              "MSCCL_DIRECT", "MSCCL_LL_SLOT_BYTES",
                                                              "MSCCL_LL128_SLOT_BYTES",
                                                              "MSCCL_CROSS_LAUNCH", "MSCCL_DIRECT_HINTS"))
    if key not in _COMMS:
        _COMMS[key] = runtime.Comm.virtual(R, device)
    return _COMMS[key]


def run_program(ir_text, inputs, count, dtype, op="sum", out_elems=None, inplace=False, device=0, fill=0xA5):
    """Load `ir_text` on R virtual ranks, run it once on `inputs` (numpy, storage dtype),
    return the per-rank outputs as numpy arrays (storage dtype)."""
    R = len(inputs)
    cs = comms(R, device)
    progs = [c.load(ir_text) for c in cs]
    try:
        raw = [np.ascontiguousarray(x) for x in inputs]
        send = [torch.from_numpy(x.view(np.uint8).copy()).to(f"cuda:{device}") for x in raw]
        if inplace:
            recv = send
        else:
            ob = (out_elems if out_elems is not None else raw[0].size) * raw[0].itemsize
            recv = [torch.full((ob,), fill, dtype=torch.uint8, device=f"cuda:{device}") for _ in range(R)]
        with runtime.group():
            for c, p, s, r in zip(cs, progs, send, recv):
                c.run(p, s, r, count, op=op, dtype=dtype)
        torch.cuda.synchronize()
        return [r.cpu().numpy().view(raw[0].dtype) for r in recv]
    finally:
        for c, p in zip(cs, progs):
            c.unload(p)
