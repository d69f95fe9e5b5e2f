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
    if dist.get_backend(group) == "gloo":
        stats = stats.cpu()
    parts = [torch.zeros_like(stats) for _ in range(dist.get_world_size(group))]
    dist.all_gather(parts, stats.contiguous(), group=group)
    return torch.cat(parts)


# ---------------------------------------------------------------- NEXT-1: global selection across GPUs
def gather_rows(tensors, group=None, counts=None):
    """all_gather of per-rank tensors whose first dimension (streams) differs
    between ranks: every tensor is padded to the largest S_r, gathered, and the
    valid rows concatenated rank-major.  Returns (gathered tensors, row offset
    of this rank).  One small exchange per chunk (<= 30k
    entries); NCCL on GPUs, gloo on CPU.  Data movement only.  counts: every
    rank's row count when the caller already knows them (they are fixed for a
    run): skips the count exchange and its host synchronisation."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
        return list(tensors), 0
    world, me = dist.get_world_size(group), dist.get_rank(group)
    dev = tensors[0].device
    if counts is None:
        counts = row_counts(tensors[0].shape[0], dev, group)
    cnts = list(counts)
    smax = max(cnts)
    out = []
    for t in tensors:
        pad = torch.zeros((smax,) + tuple(t.shape[1:]), dtype=t.dtype, device=dev)
        pad[: t.shape[0]] = t
        parts = [torch.empty_like(pad) for _ in range(world)]
        dist.all_gather(parts, pad, group=group)
        out.append(torch.cat([p[:c] for p, c in zip(parts, cnts)]))
    return out, sum(cnts[:me])


def row_counts(S, device, group=None):
    """Every rank's stream count (one all_gather; host-synchronising): compute
    once per run and pass to gather_rows / select_global_across_ranks."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
        return [int(S)]
    cnt = torch.tensor([int(S)], dtype=torch.int64, device=device)
    cnts = [torch.zeros_like(cnt) for _ in range(dist.get_world_size(group))]
    dist.all_gather(cnts, cnt, group=group)
    return [int(c.item()) for c in cnts]


def select_global_across_ranks(ctx, chunks, sid, cost, budget, fresh=False, use_res_size=False, group=None,
                               stream=None, return_all=False, n=None, device=None, shape=None, counts=None):
    """§5.2 global anchor selection over the streams of every GPU:
    (1) per-stream gains and ranks on this GPU (ns_select_anchors, Alg. 1);
    (2) all_gather of gain / rank / type / sid / cost rows (gather_rows);
    (3) ns_select_merge on the gathered rows -- the identical deterministic
    prefix on every GPU, no further exchange.  Returns this GPU's is_anchor
    [S_local, n] (device u8) for ns_enhance_streams(mode=NS_GIVEN_ANCHORS,
    anchor_in=..., cost=cost, budget=budget), and the global rank rows.
    A rank may own no streams (chunks == []): it then passes n and device, and
    still takes part in the gather and the merge.  sid / cost may be lists or
    device tensors, shape an [S, 3] device tensor of (w, h, scale), counts the
    ranks' stream counts (row_counts): a caller that passes them once-built
    keeps every host->device copy and host synchronisation out of its steps."""
    import torch
    from . import NS_TOPK_PER_STREAM
    S = len(chunks)
    n = chunks[0].n if S else int(n)
    dev = chunks[0].type.device if S else torch.device(device)
    gain = torch.zeros((S, n), dtype=torch.int64, device=dev)
    rank = torch.zeros((S, n), dtype=torch.int32, device=dev)
    anc = torch.zeros((S, n), dtype=torch.uint8, device=dev)
    if S:
        ctx.select_anchors(chunks, gain, rank, anc, stream=stream, mode=NS_TOPK_PER_STREAM, k=0, fresh=fresh,
                           use_res_size=use_res_size)
        types = torch.stack([c.type for c in chunks])
    else:
        types = torch.zeros((0, n), dtype=torch.uint8, device=dev)
    sid_t = sid if isinstance(sid, torch.Tensor) else torch.as_tensor(list(sid), dtype=torch.int32).reshape(-1).to(dev)
    cost_t = (cost if isinstance(cost, torch.Tensor) else
              torch.as_tensor(list(cost), dtype=torch.int64).reshape(-1).to(dev))
    # (w, h, scale) of every row: the anchor exchange sizes each moved frame by
    # its own stream's shape (mixed-resolution fleets)
    shape_t = shape if shape is not None else torch.as_tensor(
        [[c.w, c.h, c.scale] for c in chunks], dtype=torch.int32).reshape(-1, 3).to(dev)
    (g_all, r_all, t_all, s_all, c_all, sh_all), off = gather_rows([gain, rank, types, sid_t, cost_t, shape_t],
                                                                   group, counts)
    rank_out = torch.empty_like(r_all)
    anc_all = torch.empty_like(t_all)
    ctx.select_merge(g_all, r_all, t_all, s_all, c_all, budget, rank_out, anc_all, stream=stream)
    if return_all:  # every gathered row, for the anchor-level load balancing
        return (anc_all[off: off + S].contiguous(), rank_out[off: off + S].contiguous(),
                {"anchor": anc_all, "sid": s_all, "cost": c_all, "shape": sh_all})
    return anc_all[off: off + S].contiguous(), rank_out[off: off + S].contiguous()


# ---------------------------------------------------------------- NEXT-1: anchor-level load balancing
def plan_anchor_moves(anchors, owner, cost, world):
    """Deterministic anchor-level load balancing across GPUs (§5.2: the
    scheduler spreads the selected anchor frames' DNN work over the GPUs,
    P:205-213).  Streams stay on their GPU; single anchor SR jobs
    move.  anchors[i]: the anchor frames of gathered stream row i; owner[i]: its
    rank; cost[i]: T_DNN of one of its anchors (> 0).  Greedy: while the most
    loaded rank (lowest index on ties) has an anchor whose move to the least
    loaded rank lowers the pair's maximum, move its first such anchor in
    (row desc, frame desc) order.  Every rank computes the same plan from the
    same gathered rows.  Returns [(row, frame, src, dst)] in move order."""
    load = [0] * world
    on = [[] for _ in range(world)]
    for i, fr in enumerate(anchors):
        for f in fr:
            load[owner[i]] += cost[i]
            on[owner[i]].append((i, f))
    for r in range(world):
        on[r].sort(reverse=True)
    moves = []
    while world > 1:
        hi = min(range(world), key=lambda r: (-load[r], r))
        lo = min(range(world), key=lambda r: (load[r], r))
        pick = None
        for idx, (i, f) in enumerate(on[hi]):
            if load[lo] + cost[i] < load[hi]:
                pick = idx
                break
        if pick is None:
            break
        i, f = on[hi].pop(pick)
        load[hi] -= cost[i]
        load[lo] += cost[i]
        moves.append((i, f, hi, lo))
    return moves


def _ipc_share(t):
    """Picklable description of tensor t's memory for another process on this
    host: CUDA IPC for device memory (the peer maps it: NVLink peer memory on a
    multi-GPU node, the same GPU when ranks share one), shared memory for host
    tensors (the gloo tests)."""
    import torch.multiprocessing  # noqa: F401  (registers the tensor reductions)
    from multiprocessing.reduction import ForkingPickler
    return bytes(ForkingPickler.dumps(t))


def _ipc_open(desc):
    import pickle
    return pickle.loads(desc)


def balanced_sr_and_reconstruct(ctx, chunks, models, sid, is_anchor, hr_out, anchors_all, owner_all, sid_all, cost_all,
                                group=None, stream=None, shape_all=None, device=None, transport="nccl"):
    """SR on this GPU's share of the balanced anchor set, then reconstruction of
    this GPU's streams (ns_sr_anchors + ns_reconstruct_chunk).  anchors_all /
    owner_all / sid_all / cost_all describe every gathered stream row (host
    lists, identical on all ranks); chunks / models / sid / is_anchor / hr_out
    are this GPU's streams (models: dict sid -> Model, holding at least the
    models of the rows this GPU may serve -- per-stream weights are small and
    every GPU keeps all of them).  Exported anchors: LR out, HR back; imported
    anchors: LR in, SR here, HR out -- point-to-point over NCCL (NVLink).
    Everything is ordered on the current torch stream (stream=None), which the
    NCCL point-to-point calls synchronise with.  shape_all[i] = (w, h, scale)
    of row i (select_global_across_ranks(return_all=True)["shape"]): an
    imported anchor's LR / HR buffers take its source stream's shape.  A rank
    with no streams (chunks == []) passes `device` and still serves imports."""
    import torch
    import torch.distributed as dist
    dist_on = dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1
    world = dist.get_world_size(group) if dist_on else 1
    me = dist.get_rank(group) if dist_on else 0
    moves = plan_anchor_moves(anchors_all, owner_all, cost_all, world)
    local = {s: li for li, s in enumerate(sid)}
    exported = {(sid_all[i], f): dst for i, f, src, dst in moves if src == me}
    jobs = []
    for li, s in enumerate(sid):
        row = [i for i in range(len(sid_all)) if sid_all[i] == s][0]
        for f in anchors_all[row]:
            if (s, f) not in exported:
                jobs.append((models[s], chunks[li].lr[f], hr_out[li][f]))
    if transport == "peer" and dist_on:
        # Peer memory (§5.2 (2) without staging copies): every exporter publishes
        # its moved anchors' LR frame and HR slot; the importer maps them and runs
        # SR straight from the exporter's LR into the exporter's HR slot -- the SR
        # kernels read and write the peer's memory (k_prep_lr loads the LR frame,
        # the upsampler epilogue and border fix-up store the HR frame), so the
        # transfer rides inside the kernels instead of separate NCCL copies.
        if chunks and chunks[0].lr.is_cuda:
            torch.cuda.current_stream().synchronize()   # this rank's inputs and HR slots are settled
        offer = {}
        for i, f, src, dst in moves:
            if src == me:
                s = sid_all[i]
                offer[(i, f)] = (_ipc_share(chunks[local[s]].lr[f]), _ipc_share(hr_out[local[s]][f]))
        offers = [None] * world
        dist.all_gather_object(offers, offer, group=group)
        mapped = []
        for i, f, src, dst in moves:
            if dst == me:
                lr, hr = (_ipc_open(d) for d in offers[src][(i, f)])
                mapped.append((lr, hr))
                jobs.append((models[sid_all[i]], lr, hr))
        if jobs:
            ctx.sr_anchors(jobs, stream=stream)
            if mapped and mapped[0][0].is_cuda:
                (stream if stream is not None else torch.cuda.current_stream()).synchronize()
        dist.barrier(group=group)             # every moved anchor's HR is in its owner's slot
        del mapped
        if chunks:
            ctx.reconstruct_chunk(chunks, is_anchor, hr_out, stream=stream)
        return moves
    if dist_on and moves and dist.get_backend(group) == "gloo" and (
            (chunks and chunks[0].lr.is_cuda) or (device is not None and torch.device(device).type == "cuda")):
        raise ValueError("point-to-point copies of device tensors need the nccl backend; "
                         "with gloo use transport='peer'")
    imports = []
    ops = []
    for i, f, src, dst in moves:          # LR out / in, in the global move order on every rank
        s = sid_all[i]
        if src == me:
            ops.append(dist.P2POp(dist.isend, chunks[local[s]].lr[f].contiguous(), dst, group))
        elif dst == me:
            if shape_all is not None:
                w, h, sc = (int(v) for v in shape_all[i])
            else:  # uniform fleets: every row has this rank's shape
                w, h, sc = chunks[0].w, chunks[0].h, chunks[0].scale
            dev = chunks[0].lr.device if chunks else torch.device(device)
            lr = torch.empty((3, h, w), dtype=torch.uint8, device=dev)
            hr = torch.empty((3, sc * h, sc * w), dtype=torch.uint8, device=dev)
            imports.append((i, f, src, lr, hr))
            ops.append(dist.P2POp(dist.irecv, lr, src, group))
    if ops:
        for rq in dist.batch_isend_irecv(ops):
            rq.wait()
    for i, f, src, lr, hr in imports:
        jobs.append((models[sid_all[i]], lr, hr))
    if jobs:
        ctx.sr_anchors(jobs, stream=stream)
    ops = []
    for i, f, src, dst in moves:          # HR back
        s = sid_all[i]
        if dst == me:
            hr = [x for x in imports if x[0] == i and x[1] == f][0][4]
            ops.append(dist.P2POp(dist.isend, hr, src, group))
        elif src == me:
            ops.append(dist.P2POp(dist.irecv, hr_out[local[s]][f], dst, group))
    if ops:
        for rq in dist.batch_isend_irecv(ops):
            rq.wait()
    if chunks:
        ctx.reconstruct_chunk(chunks, is_anchor, hr_out, stream=stream)
    return moves
