"""Multi-GPU host logic on CPU: LPT sharding and the gloo (world_size 2)
stats gather / max-over-ranks used by bench.py after the timed region."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sigcomm_yeolkjyh22_b200 import shard


def test_flop_model_matches_survey():
    assert shard.sr_flop_per_lr_px(8, 32, 3) == shard.SR_FLOP_PER_LR_PX[(8, 32, 3)]


def test_lpt_balanced_and_complete():
    # c5-like mix: half 720p->4K, half 360p->1080p
    costs = [shard.stream_cost(1280, 720, 3, 60, 5) if i % 2 == 0 else shard.stream_cost(640, 360, 3, 60, 5)
             for i in range(512)]
    for world in (1, 2, 4, 8):
        parts = shard.lpt_shard(costs, world)
        flat = sorted(i for p in parts for i in p)
        assert flat == list(range(512))
        loads = [sum(costs[i] for i in p) for p in parts]
        assert max(loads) - min(loads) <= max(costs) + 1e-12
        # deterministic
        assert parts == shard.lpt_shard(costs, world)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        local = torch.full((3, 8), float(rank), dtype=torch.float64)
        local[:, 0] = torch.arange(3, dtype=torch.float64) + 10 * rank
        allst = shard.gather_stats(local)
        tmax = shard.max_over_ranks(1.5 + rank)
        q.put((rank, allst.tolist(), tmax))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_gather_and_max():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, allst, tmax in res:
        assert tmax == 2.5
        t = torch.tensor(allst)
        assert t.shape == (6, 8)
        assert t[:3, 0].tolist() == [0.0, 1.0, 2.0] and t[3:, 0].tolist() == [10.0, 11.0, 12.0]
        assert (t[3:, 1:] == 1.0).all() and (t[:3, 1:] == 0.0).all()


# ---------------------------------------------------------------- NEXT-1 host logic (gloo, world 2)
def _merge_worker(rank, world, port, q):
    """Each rank owns an unequal, interleaved subset of 7 streams; it computes
    its streams' gains with the oracle (standing in for ns_select_anchors),
    gathers the rows with shard.gather_rows, and runs the oracle merge on the
    gathered rows.  Every rank must get the selection of select_global over
    all streams, and its own rows at the returned offset."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import select as S
        streams, cost = _merge_streams()
        mine = [i for i in range(len(streams)) if (i % 3 == 0) == (rank == 0)]   # 3 vs 4 streams
        n = len(streams[0][0])
        gain = torch.tensor([S.select_topk(*streams[i], 0)[0] for i in mine], dtype=torch.int64)
        rk = torch.tensor([S.select_topk(*streams[i], 0)[1] for i in mine], dtype=torch.int32)
        ty = torch.tensor([streams[i][0] for i in mine], dtype=torch.uint8)
        sid = torch.tensor(mine, dtype=torch.int32)
        co = torch.tensor([cost[i] for i in mine], dtype=torch.int64)
        (g, r, t, s, c), off = shard.gather_rows([gain, rk, ty, sid, co])
        assert g.shape == (len(streams), n) and t.dtype == torch.uint8
        _, a = S.merge_gathered(t.tolist(), g.tolist(), s.tolist(), c.tolist(), 9)
        q.put((rank, s.tolist(), off, len(mine), a, g.tolist()))
    finally:
        dist.destroy_process_group()


def _merge_streams():
    import random
    rng = random.Random(3)
    from oracle import select as S
    streams = []
    for _ in range(7):
        types = [S.KEY] + [rng.choice((S.NORMAL, S.NORMAL, S.ALTREF)) for _ in range(9)]
        streams.append((types, [rng.randint(1, 50) for _ in range(10)]))
    return streams, [rng.randint(1, 3) for _ in range(7)]


def test_gloo_world2_global_selection_rows():
    from oracle import select as S
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_merge_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    streams, cost = _merge_streams()
    gains_all, _, anc_all = S.select_global(streams, cost, 9)
    (r0, sid0, off0, n0, a0, g0), (r1, sid1, off1, n1, a1, g1) = res
    assert sid0 == sid1 == [0, 3, 6, 1, 2, 4, 5]          # rank-major rows, unequal counts
    assert (off0, n0, off1, n1) == (0, 3, 3, 4)
    assert g0 == g1 == [gains_all[i] for i in sid0]         # gathered gains are every stream's
    assert a0 == a1 == [anc_all[i] for i in sid0]           # = global selection over all streams


# ---------------------------------------------------------------- NEXT-1 anchor-level load balancing
def test_plan_anchor_moves_balances_and_is_deterministic():
    import random
    rng = random.Random(4)
    for world in (1, 2, 4, 8):
        for _ in range(20):
            rows = rng.randint(world, 40)
            owner = [rng.randrange(world) for _ in range(rows)]
            cost = [rng.choice((1, 4)) for _ in range(rows)]      # 360p vs 720p anchor
            anchors = [sorted(rng.sample(range(60), rng.randint(0, 9))) for _ in range(rows)]
            moves = shard.plan_anchor_moves(anchors, owner, cost, world)
            assert moves == shard.plan_anchor_moves(anchors, owner, cost, world)
            load = [0] * world
            for i, fr in enumerate(anchors):
                load[owner[i]] += cost[i] * len(fr)
            before = max(load)
            seen = set()
            for i, f, src, dst in moves:
                assert f in anchors[i] and (i, f) not in seen and src != dst
                seen.add((i, f))
                load[src] -= cost[i]
                load[dst] += cost[i]
            assert max(load) <= before
            # no single remaining move (an anchor moves at most once) from the max
            # to the min rank lowers the max
            hi, lo = load.index(max(load)), load.index(min(load))
            unmoved = [(i, f) for i, fr in enumerate(anchors) for f in fr if (i, f) not in seen and owner[i] == hi]
            assert all(load[lo] + cost[i] >= load[hi] for i, f in unmoved)
            if world == 1:
                assert moves == []


class _FakeCtx:
    """Stands in for ns.Context on CPU: 'SR' = nearest x2 upsample + model id."""
    def __init__(self):
        self.sr_calls, self.recon_calls = 0, 0

    def sr_anchors(self, jobs, stream=None):
        self.sr_calls += 1
        for m, lr, hr in jobs:
            hr.copy_((lr.repeat_interleave(2, 1).repeat_interleave(2, 2).int() + m) % 256)

    def reconstruct_chunk(self, chunks, is_anchor, hr_out, stream=None):
        self.recon_calls += 1


def _lb_worker(rank, world, port, q, transport="nccl"):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    if transport == "peer":   # host tensors shared by file name (the CUDA analogue is CUDA IPC)
        mp.set_sharing_strategy("file_system")
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from types import SimpleNamespace
        n, h, w = 6, 4, 8
        S_tot = 5
        owner_all = [0, 0, 0, 0, 1]                     # rank 0 holds 4 streams, rank 1 one
        sid_all = list(range(S_tot))
        cost_all = [1] * S_tot
        anchors_all = [[0, 3], [0, 2], [0], [0, 5], [0]]
        mine = [i for i in range(S_tot) if owner_all[i] == rank]
        g = torch.Generator().manual_seed(9)
        lr_all = torch.randint(0, 256, (S_tot, n, 3, h, w), generator=g, dtype=torch.int32).to(torch.uint8)
        chunks = [SimpleNamespace(lr=lr_all[i], h=h, w=w, scale=2) for i in mine]
        hr_out = [[torch.zeros((3, 2 * h, 2 * w), dtype=torch.uint8) for _ in range(n)] for _ in mine]
        models = {s: 10 + s for s in sid_all}
        ia = torch.zeros((len(mine), n), dtype=torch.uint8)
        ctx = _FakeCtx()
        moves = shard.balanced_sr_and_reconstruct(ctx, chunks, models, mine, ia, hr_out, anchors_all, owner_all,
                                                  sid_all, cost_all, transport=transport)
        ok = True
        for li, s in enumerate(mine):
            for f in anchors_all[s]:
                exp = (lr_all[s, f].repeat_interleave(2, 1).repeat_interleave(2, 2).int() + models[s]) % 256
                ok &= bool(torch.equal(hr_out[li][f], exp.to(torch.uint8)))
        q.put((rank, moves, ok, ctx.recon_calls))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("transport", ["nccl", "peer"])
def test_gloo_world2_balanced_sr_exchange(transport):
    """transport nccl: point-to-point copies; peer: the importer writes the
    exporter's HR slots through a mapping of its memory (no copies)."""
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_lb_worker, args=(r, world, port, q, transport)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    (r0, m0, ok0, rc0), (r1, m1, ok1, rc1) = res
    assert m0 == m1 and len(m0) == 3                        # loads 7 / 1 -> 4 / 4
    assert all(src == 0 and dst == 1 for _, _, src, dst in m0)
    assert ok0 and ok1                                      # every anchor's HR is its own stream's SR
    assert rc0 == rc1 == 1


def _lb_worker_mixed(rank, world, port, q, transport="nccl"):
    """Mixed resolutions (c5-like fleets) and a rank that owns no stream: the
    imported anchors' buffers take their source stream's shape (shape_all)."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    if transport == "peer":
        mp.set_sharing_strategy("file_system")
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from types import SimpleNamespace
        n = 6
        shapes = [(8, 4, 2), (16, 8, 2), (8, 4, 2), (24, 8, 2)]   # (w, h, scale) per stream
        S_tot = len(shapes)
        owner_all = [0] * S_tot                         # rank 1 owns nothing
        sid_all = list(range(S_tot))
        cost_all = [1, 4, 1, 6]
        anchors_all = [[0, 3], [0, 2], [0], [0, 5]]
        mine = [i for i in range(S_tot) if owner_all[i] == rank]
        g = torch.Generator().manual_seed(11)
        lr_all = [torch.randint(0, 256, (n, 3, h, w), generator=g, dtype=torch.int32).to(torch.uint8)
                  for (w, h, _) in shapes]
        chunks = [SimpleNamespace(lr=lr_all[i], w=shapes[i][0], h=shapes[i][1], scale=2) for i in mine]
        hr_out = [[torch.zeros((3, 2 * shapes[i][1], 2 * shapes[i][0]), dtype=torch.uint8) for _ in range(n)]
                  for i in mine]
        models = {s: 20 + s for s in sid_all}
        ia = torch.zeros((len(mine), n), dtype=torch.uint8)
        ctx = _FakeCtx()
        moves = shard.balanced_sr_and_reconstruct(ctx, chunks, models, mine, ia, hr_out, anchors_all, owner_all,
                                                  sid_all, cost_all, shape_all=shapes, device="cpu", transport=transport)
        ok = True
        for li, s in enumerate(mine):
            for f in anchors_all[s]:
                exp = (lr_all[s][f].repeat_interleave(2, 1).repeat_interleave(2, 2).int() + models[s]) % 256
                ok &= bool(torch.equal(hr_out[li][f], exp.to(torch.uint8)))
        q.put((rank, moves, ok, ctx.recon_calls))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("transport", ["nccl", "peer"])
def test_gloo_world2_balanced_mixed_shapes_empty_rank(transport):
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_lb_worker_mixed, args=(r, world, port, q, transport)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    (r0, m0, ok0, rc0), (r1, m1, ok1, rc1) = res
    assert m0 == m1 and len(m0) > 0
    assert {shapes_i for shapes_i, *_ in m0} & {1, 3}       # large-frame rows moved too
    assert ok0 and ok1
    assert (rc0, rc1) == (1, 0)                             # the empty rank reconstructs nothing
