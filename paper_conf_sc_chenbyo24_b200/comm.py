"""Process-group plumbing for the one-time IPC-handle exchange.

The C ABI takes an all-gather callback; these build one from torch.distributed
(one process per GPU, NCCL or gloo) or from threads (single-process simulation of
G ranks, used by the 1-GPU tests).  Nothing here is on the per-forward path.
"""
from __future__ import annotations

import threading
from typing import Callable, List


def torch_allgather(group=None) -> Callable[[bytes], bytes]:
    import torch
    import torch.distributed as dist

    def ag(b: bytes) -> bytes:
        world = dist.get_world_size(group)
        t = torch.frombuffer(bytearray(b), dtype=torch.uint8)
        if dist.get_backend(group) == "nccl":
            t = t.cuda()
            out = torch.empty(world * len(b), dtype=torch.uint8, device=t.device)
            dist.all_gather_into_tensor(out, t, group=group)
            return out.cpu().numpy().tobytes()
        outs = [torch.empty_like(t) for _ in range(world)]
        dist.all_gather(outs, t, group=group)
        return b"".join(o.numpy().tobytes() for o in outs)

    return ag


class LocalGroup:
    """In-process all-gather for G simulated ranks driven by G host threads."""

    def __init__(self, world_size: int):
        self.G = world_size
        self._barrier = threading.Barrier(world_size)
        self._buf: List[bytes] = [b""] * world_size

    def allgather_for(self, rank: int) -> Callable[[bytes], bytes]:
        def ag(b: bytes) -> bytes:
            self._buf[rank] = b
            self._barrier.wait()
            out = b"".join(self._buf)
            self._barrier.wait()
            return out

        return ag


def run_ranks(world_size: int, fn: Callable[[int], object]) -> list:
    """Run fn(rank) on `world_size` threads (collective registration in simulation)."""
    res: list = [None] * world_size
    err: list = []

    def body(r):
        try:
            res[r] = fn(r)
        except BaseException as e:  # surfaced below
            err.append(e)

    th = [threading.Thread(target=body, args=(r,)) for r in range(world_size)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    if err:
        raise err[0]
    return res
