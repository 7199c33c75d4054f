"""One process per GPU: torch.distributed plumbing around the C ABI.

The spread's device list is the job's ranks in order (list position = rank,
PAPER.md:101); each process owns the chunks of its position
(somier_init_local). The fused halo exchange needs every neighbour chunk's
device memory: the processes swap CUDA IPC blobs (somier_ipc_export) with one
all_gather_object and open them (somier_ipc_connect). From then on the step
runs entirely in the kernels: boundary planes are stored into the neighbour's
halo slot over NVLink and completion is signalled with a device flag that the
neighbour's stream waits on -- no host round trip and no NCCL call per step.
Stats are combined exactly from the per-process int128 partials.
"""
from __future__ import annotations

import os
from typing import List, Optional, Sequence

from .somier import Somier, SomierParams, Stats, combine_stats
from .spread import Spread


def env_rank() -> tuple:
    """(rank, world_size, local_rank) from the torchrun environment (defaults: 0, 1, 0)."""
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", str(rank)))
    return rank, world, local


def all_gather_bytes(blob: bytes, group=None) -> List[bytes]:
    import torch.distributed as dist

    out: List[Optional[bytes]] = [None] * dist.get_world_size(group)
    dist.all_gather_object(out, blob, group=group)
    return [bytes(b) for b in out]


def all_gather_obj(obj, group=None) -> list:
    """Every rank's picklable `obj`, in rank order (plumbing for bench reports)."""
    import torch.distributed as dist

    out: List[Optional[object]] = [None] * dist.get_world_size(group)
    dist.all_gather_object(out, obj, group=group)
    return out


def connect(s: Somier, group=None) -> None:
    """Exchange IPC blobs with every rank and open the neighbours' memory."""
    import torch.distributed as dist

    blobs = all_gather_bytes(s.ipc_export(), group)
    s.ipc_connect(blobs)
    dist.barrier(group)


def open_local(params: SomierParams, chunk: int = 0, group=None, cuda_device: Optional[int] = None) -> Somier:
    """Create this rank's part of a grid spread over all ranks (devices(0..world-1)).
    Fused / copy exchange: the ranks swap CUDA IPC blobs; NCCL exchange
    (params.exchange == EXCHANGE_NCCL): rank 0's ncclUniqueId is shared and every
    rank joins the communicator (somier_nccl_connect)."""
    import ctypes

    import torch.distributed as dist

    from . import _native as N

    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    spread = Spread(list(range(world)), 1, params.n[0] - 2, chunk=chunk)
    s = Somier(spread, params, device_pos=rank, cuda_device=rank if cuda_device is None else cuda_device)
    if params.exchange == N.EXCHANGE_NCCL:
        uid = ctypes.create_string_buffer(128)
        if rank == 0:
            N.check(N.lib().somier_nccl_unique_id(uid), "somier_nccl_unique_id")
        ids = all_gather_bytes(uid.raw, group)
        N.check(N.lib().somier_nccl_connect(s._h, ctypes.create_string_buffer(ids[0], 128), world),
                "somier_nccl_connect")
        dist.barrier(group)
    else:
        connect(s, group)
    return s


def gather_stats(s: Somier, group=None) -> Stats:
    """Exact global stats: per-rank int128 partials combined by somier_stats_combine."""
    import torch.distributed as dist

    mine = s.stats()
    parts: List[Optional[Stats]] = [None] * dist.get_world_size(group)
    dist.all_gather_object(parts, mine, group=group)
    return combine_stats(parts, s.params)


def gather_stats_history(s: Somier, first_step: int, count: int, group=None) -> List[Stats]:
    """Exact global stats of steps first_step .. first_step+count-1 (every
    rank's somier_stats_history partials combined step by step)."""
    mine = s.stats_history(first_step, count)
    parts = all_gather_obj(mine, group)
    return [combine_stats([p[i] for p in parts], s.params) for i in range(count)]


def combine_partials(parts: Sequence[Stats], params: SomierParams) -> Stats:
    return combine_stats(parts, params)
