"""Multi-GPU sharded generation: one process per GPU.

Every rank expands the small replicated prefix and a balanced contiguous slice of the
cut level on its own GPU (``atf_space_generate_shard``); the only exchange is an
all-gather of the per-(group, level) node counts (int64, < 1 KB) through
``torch.distributed`` — NCCL over NVLink/NVSwitch on GPUs, gloo on CPU tests — after
which ``atf_space_finalize_shard`` turns them into this rank's global offsets and the
global group sizes.
"""
from __future__ import annotations

from typing import List, Optional

import torch
import torch.distributed as dist


def all_gather_counts(counts: List[int], group=None, device: Optional[torch.device] = None) -> List[List[int]]:
    """All-gather one int64 vector per rank -> [world][n] (rank-major) on every rank."""
    world = dist.get_world_size(group)
    if device is None:
        device = torch.device("cuda", torch.cuda.current_device()) \
            if dist.get_backend(group) == "nccl" else torch.device("cpu")
    t = torch.tensor(counts, dtype=torch.int64, device=device)
    out = torch.empty(world * t.numel(), dtype=torch.int64, device=device)
    dist.all_gather_into_tensor(out, t, group=group)
    return out.view(world, -1).cpu().tolist()


def generate_sharded(space, group=None) -> List[List[int]]:
    """Generate this rank's shard of `space` and finalize it with the other ranks' counts.
    Returns the gathered counts ([world][n])."""
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    counts = space.generate_shard(rank, world)
    allc = all_gather_counts(counts, group)
    space.finalize_shard(allc)
    return allc
