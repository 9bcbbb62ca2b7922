"""Multi-GPU generation: one process per GPU.

``generate_balanced`` (atf_space_generate_dist, the default): every level is redistributed —
rank r expands the parent slice [r F / N, (r + 1) F / N) of the previous level — with one small
all-gather per level round through ``torch.distributed`` (NCCL over NVLink / NVSwitch on GPUs,
gloo on CPU tests); the parent slices move between GPUs as CUDA IPC peer copies inside the
library.  ``generate_sharded`` (atf_space_generate_shard + finalize_shard): the older static
partition of one cut level, one all-gather at the end.  ``virtual_ranks`` runs N spaces of one
process as ranks (tests, the one-GPU scaling prediction in bench.py).
"""
from __future__ import annotations

import threading
import time

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


def _allgather_bytes(data: bytes, group=None) -> bytes:
    world = dist.get_world_size(group)
    device = torch.device("cuda", torch.cuda.current_device()) if dist.get_backend(group) == "nccl" \
        else torch.device("cpu")
    t = torch.frombuffer(bytearray(data), dtype=torch.uint8).to(device)
    out = torch.empty(world * t.numel(), dtype=torch.uint8, device=device)
    dist.all_gather_into_tensor(out, t, group=group)
    return out.cpu().numpy().tobytes()


def generate_balanced(space, group=None) -> None:
    """Balanced generation of this rank's part of `space` (every level redistributed)."""
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    space.generate_dist(rank, world, lambda b: _allgather_bytes(b, group))


class VirtualAllGather:
    """All-gather among `world` threads of one process (ranks = spaces on one GPU).  With
    `serialize`, only one rank works between two all-gathers at a time and the host time of
    each rank's round is recorded (`round_s[rank][round]`): per-rank level times without the
    ranks sharing the GPU."""

    def __init__(self, world: int, serialize: bool = False):
        self.world = world
        self.barrier = threading.Barrier(world)
        self.slots = [b""] * world
        self.serialize = serialize
        self.lock = threading.Lock()
        self.round_s = [[] for _ in range(world)]
        self.calls = [0] * world
        self._t0 = [0.0] * world

    def start(self, rank: int):
        if self.serialize:
            self.lock.acquire()
            self._t0[rank] = time.perf_counter()

    def __call__(self, rank: int, data: bytes) -> bytes:
        self.calls[rank] += 1
        if self.serialize:
            self.round_s[rank].append(time.perf_counter() - self._t0[rank])
            self.lock.release()
        self.slots[rank] = data
        self.barrier.wait()
        out = b"".join(self.slots)
        self.barrier.wait()
        if self.serialize:
            self.lock.acquire()
            self._t0[rank] = time.perf_counter()
        return out

    def finish(self, rank: int):
        if self.serialize:
            self.round_s[rank].append(time.perf_counter() - self._t0[rank])
            self.lock.release()


def virtual_ranks(spaces, serialize: bool = False) -> VirtualAllGather:
    """generate_dist on every space of `spaces` (rank = position), in threads of this process."""
    world = len(spaces)
    vag = VirtualAllGather(world, serialize)
    errs = []

    def run(r):
        try:
            torch.cuda.set_device(spaces[r]._device)
            vag.start(r)
            spaces[r].generate_dist(r, world, lambda b: vag(r, b))
            torch.cuda.synchronize()
            vag.finish(r)
        except Exception as ex:  # noqa: BLE001
            errs.append(ex)
            vag.barrier.abort()

    th = [threading.Thread(target=run, args=(r,)) for r in range(world)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    if errs:
        raise errs[0]
    return vag
