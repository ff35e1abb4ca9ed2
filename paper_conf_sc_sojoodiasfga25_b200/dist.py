"""torch.distributed bootstrap for multi-rank contexts (plumbing only).

The library needs one collective primitive at mp_init / mp_finalize: an all-gather
of a few hundred bytes per rank (IPC handles, job id, barriers).  This module
adapts torch.distributed (gloo or NCCL) to the C callback `mp_allgather_fn`.
"""
from __future__ import annotations

import ctypes
import sys
import traceback

from .mp import Context


def torch_allgather(group=None):
    import torch.distributed as dist

    def ag(_user, inp, out, nbytes):
        try:
            data = ctypes.string_at(inp, nbytes)
            objs = [None] * dist.get_world_size(group)
            dist.all_gather_object(objs, data, group=group)
            blob = b"".join(objs)
            if len(blob) != nbytes * len(objs):
                return -1
            ctypes.memmove(out, blob, len(blob))
            return 0
        except Exception:  # never let an exception cross the C boundary
            traceback.print_exc(file=sys.stderr)
            return -1

    return ag


def context_from_dist(group=None, **kw) -> Context:
    """Create a collective mp context over the current torch.distributed group."""
    import torch.distributed as dist
    return Context(rank=dist.get_rank(group), world=dist.get_world_size(group),
                   allgather=torch_allgather(group), **kw)
