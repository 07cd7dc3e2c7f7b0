"""One process per GPU: build a connected communicator from a torch.distributed group.

Host-side plumbing only (the handle exchange); the collectives themselves never touch
torch.distributed or NCCL. Each rank exports the CUDA IPC handle of its shared region
(mscclCommExportHandle), the handles are all-gathered over the process group (any
backend — gloo, or NCCL used as plumbing), and every rank opens its peers' regions
(mscclCommConnect).
"""


def exchange_handles(handle, group=None):
    """All-gather this rank's handle bytes; returns the list in rank order."""
    import torch.distributed as dist
    world = dist.get_world_size(group)
    out = [None] * world
    dist.all_gather_object(out, bytes(handle), group=group)
    size = len(out[0])
    if any(not isinstance(h, (bytes, bytearray)) or len(h) != size for h in out):
        raise RuntimeError("inconsistent communicator handles across ranks")
    return out


def connect(comm, group=None):
    """Export, exchange and connect `comm` (an object with export_handle()/connect())."""
    comm.connect(exchange_handles(comm.export_handle(), group))
    return comm


def init_from_process_group(device, group=None):
    """mscclCommInitRank + exchange + connect for the calling process's rank."""
    import torch.distributed as dist
    from .runtime import Comm
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    return connect(Comm.init_rank(world, rank, device), group)


def register(comm, tensor, group=None):
    """Collective buffer registration for direct placement across processes (reading R15b):
    mscclCommRegister + exchange of the descriptors + mscclRegConnect on every rank, then a
    barrier so that no rank publishes the buffer before every peer has mapped it."""
    import torch.distributed as dist
    reg = comm.register(tensor)
    reg.connect(exchange_handles(reg.export(), group))
    dist.barrier(group)
    return reg
