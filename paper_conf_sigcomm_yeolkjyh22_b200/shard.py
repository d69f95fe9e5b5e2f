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


# ---------------------------------------------------------------- NEXT-1: global selection across GPUs
def gather_rows(tensors, group=None):
    """all_gather of per-rank tensors whose first dimension (streams) differs
    between ranks: every tensor is padded to the largest S_r, gathered, and the
    valid rows concatenated rank-major.  Returns (gathered tensors, row offset
    of this rank).  One small exchange per chunk (<= 30k
    entries); NCCL on GPUs, gloo on CPU.  Data movement only."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
        return list(tensors), 0
    world, me = dist.get_world_size(group), dist.get_rank(group)
    dev = tensors[0].device
    cnt = torch.tensor([tensors[0].shape[0]], dtype=torch.int64, device=dev)
    cnts = [torch.zeros_like(cnt) for _ in range(world)]
    dist.all_gather(cnts, cnt, group=group)
    cnts = [int(c.item()) for c in cnts]
    smax = max(cnts)
    out = []
    for t in tensors:
        pad = torch.zeros((smax,) + tuple(t.shape[1:]), dtype=t.dtype, device=dev)
        pad[: t.shape[0]] = t
        parts = [torch.empty_like(pad) for _ in range(world)]
        dist.all_gather(parts, pad, group=group)
        out.append(torch.cat([p[:c] for p, c in zip(parts, cnts)]))
    return out, sum(cnts[:me])


def select_global_across_ranks(ctx, chunks, sid, cost, budget, fresh=False, use_res_size=False, group=None,
                               stream=None):
    """§5.2 global anchor selection over the streams of every GPU:
    (1) per-stream gains and ranks on this GPU (ns_select_anchors, Alg. 1);
    (2) all_gather of gain / rank / type / sid / cost rows (gather_rows);
    (3) ns_select_merge on the gathered rows -- the identical deterministic
    prefix on every GPU, no further exchange.  Returns this GPU's is_anchor
    [S_local, n] (device u8) for ns_enhance_streams(mode=NS_GIVEN_ANCHORS,
    anchor_in=..., cost=cost, budget=budget), and the global rank rows."""
    import torch
    from . import NS_TOPK_PER_STREAM
    S, n = len(chunks), chunks[0].n
    dev = chunks[0].type.device
    gain = torch.empty((S, n), dtype=torch.int64, device=dev)
    rank = torch.empty((S, n), dtype=torch.int32, device=dev)
    anc = torch.empty((S, n), dtype=torch.uint8, device=dev)
    ctx.select_anchors(chunks, gain, rank, anc, stream=stream, mode=NS_TOPK_PER_STREAM, k=0, fresh=fresh,
                       use_res_size=use_res_size)
    types = torch.stack([c.type for c in chunks])
    sid_t = torch.as_tensor(list(sid), dtype=torch.int32).to(dev)
    cost_t = torch.as_tensor(list(cost), dtype=torch.int64).to(dev)
    (g_all, r_all, t_all, s_all, c_all), off = gather_rows([gain, rank, types, sid_t, cost_t], group)
    rank_out = torch.empty_like(r_all)
    anc_all = torch.empty_like(t_all)
    ctx.select_merge(g_all, r_all, t_all, s_all, c_all, budget, rank_out, anc_all, stream=stream)
    return anc_all[off: off + S].contiguous(), rank_out[off: off + S].contiguous()
