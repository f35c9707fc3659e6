"""Frame-sharded multi-GPU runs.

Frames are independent units: rank r of P takes the contiguous global frames
[floor(r*n/P), floor((r+1)*n/P)), runs the whole path locally (K1..K4), and the only collective
is the gather of the detection lists: all_gather of the per-rank counts, then all_gather of the
count-padded [max, 10] int32 detection tensors (NCCL over NVLink on GPUs, gloo on CPU tests).
Concatenation in rank order is already global frame order.  One process per GPU; torch is the
plumbing (process group, device tensors); the detection work stays in libfd.so.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

FRAME_COL = 0


def shard(n_total: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous frame range [start, end) of `rank`."""
    if world < 1 or not (0 <= rank < world):
        raise ValueError("bad rank/world")
    return (rank * n_total) // world, ((rank + 1) * n_total) // world


def globalize(dets: torch.Tensor, frame_offset: int) -> torch.Tensor:
    """Local frame indices -> global ones (column 0 of the [n, 10] int32 records)."""
    if frame_offset and dets.numel():
        dets = dets.clone()
        dets[:, FRAME_COL] += frame_offset
    return dets


def gather_detections(dets: torch.Tensor, group=None) -> torch.Tensor:
    """All-gather variable-length [n_r, 10] int32 detection tensors; returns the concatenation
    in rank order on every rank.  Two collectives: counts, then padded payloads.  With a backend
    that cannot move device tensors (gloo) the payload goes through host memory and the result
    comes back to the caller's device."""
    world = dist.get_world_size(group)
    if dets.is_cuda and dist.get_backend(group) != "nccl":
        return gather_detections(dets.cpu(), group).to(dets.device)
    dev = dets.device
    cnt = torch.tensor([dets.shape[0]], dtype=torch.int64, device=dev)
    counts = [torch.zeros_like(cnt) for _ in range(world)]
    dist.all_gather(counts, cnt, group=group)
    counts = [int(c.item()) for c in counts]
    mx = max(max(counts), 1)
    pad = torch.zeros((mx, dets.shape[1] if dets.dim() == 2 else 10), dtype=torch.int32, device=dev)
    if dets.shape[0]:
        pad[: dets.shape[0]] = dets
    bufs = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(bufs, pad, group=group)
    return torch.cat([b[:c] for b, c in zip(bufs, counts)], dim=0)
