"""Stream sharding across GPUs and the post-run stats gather.

Streams are independent (each stream's reuse chain, selection and SR jobs stay
on one device), so N GPUs = N shards with NO collective on the hot path
(PAPER.md P:213 distributes anchor work per instance; P:259 the instances talk
over gRPC only).  Host-side logic only; the hot path runs in the C ABI.

  stream_cost  analytic per-stream cost of one chunk (SR FLOPs on k anchors at
               the measured tensor rate + reconstruction bytes at HBM rate)
  lpt_shard    longest-processing-time greedy assignment of streams to ranks
  gather_stats all_gather of the per-stream [S_local, 8] stats after timing
  max_over_ranks  the job time is the slowest rank's
"""
from __future__ import annotations

import heapq
from typing import Sequence

SR_FLOP_PER_LR_PX = {(8, 32, 3): 496_512}  # SURVEY.md §8(d), defined convs only


def sr_flop_per_lr_px(B: int, C: int, s: int) -> float:
    """FLOPs of the SR net per LR pixel: head 54C + 2B body + end 18C^2 each +
    up 18 s^2 C^2 + tail 54 C s^2 (3x3 convs, 2 FLOP per MAC)."""
    return 54 * C + (2 * B + 1) * 18 * C * C + 18 * s * s * C * C + 54 * C * s * s


def stream_cost(w: int, h: int, s: int, n: int, k: int, B: int = 8, C: int = 32,
                tflops: float = 1398.0, hbm_gbs: float = 6454.0) -> float:
    """Seconds of one chunk of one stream at the given rates (a ranking key)."""
    sr = k * w * h * sr_flop_per_lr_px(B, C, s) / (tflops * 1e12)
    recon = (n - k) * (w * h * s * s * 6.0 + w * h * 6.0) / (hbm_gbs * 1e9)
    return sr + recon


def lpt_shard(costs: Sequence[float], world: int) -> list[list[int]]:
    """LPT greedy: streams in decreasing cost, each to the least-loaded rank.
    Deterministic (ties -> lower stream index, lower rank)."""
    order = sorted(range(len(costs)), key=lambda i: (-costs[i], i))
    heap = [(0.0, r) for r in range(world)]
    heapq.heapify(heap)
    out: list[list[int]] = [[] for _ in range(world)]
    for i in order:
        load, r = heapq.heappop(heap)
        out[r].append(i)
        heapq.heappush(heap, (load + costs[i], r))
    return [sorted(x) for x in out]


def max_over_ranks(value: float, group=None) -> float:
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
        return float(value)
    dev = "cuda" if dist.get_backend(group) == "nccl" else "cpu"
    t = torch.tensor([float(value)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def gather_stats(stats, group=None):
    """all_gather of equally sized [S_local, 8] fp64 tensors -> [world*S_local, 8]
    (rank-major).  Runs after the timed region; NCCL on GPUs, gloo on CPU."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
        return stats
    parts = [torch.zeros_like(stats) for _ in range(dist.get_world_size(group))]
    dist.all_gather(parts, stats.contiguous(), group=group)
    return torch.cat(parts)
