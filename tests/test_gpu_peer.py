"""NEXT-1 anchor-level load balancing with the peer-memory transport
(shard.balanced_sr_and_reconstruct(transport="peer")): two ranks (gloo for the
host collectives) share this one GPU; the importing rank maps the exporting
rank's LR frames and HR slots through CUDA IPC and its SR kernels read and
write them directly -- on a multi-GPU node the same mappings are NVLink peer
memory.  The result must equal the one-call NS_GIVEN_ANCHORS path byte for
byte."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _peer_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synth
        import paper_conf_sigcomm_yeolkjyh22_b200 as ns
        from paper_conf_sigcomm_yeolkjyh22_b200 import shard
        from helpers import alloc_hr, dev_chunk
        dev = "cuda:0"
        torch.cuda.set_device(0)
        ctx = ns.Context(0, pool_bytes=2 << 30)
        S, n = 4, 8
        cs = [synth.make_chunk(7700 + s, 48, 24, 2, n, types=synth.default_types(n, 4)) for s in range(S)]
        models = {}
        for s in range(S):
            m = ctx.model(1, 16, 2)
            m.set_weights(synth.make_weights(90 + s, 1, 16, 2))
            models[s] = m
        owner_all = [0] * S                       # rank 1 owns no stream: every move goes 0 -> 1
        anchors_all = [[0, 3], [0, 5], [0, 2, 6], [0]]
        anc_full = torch.zeros((S, n), dtype=torch.uint8, device=dev)
        for s in range(S):
            anc_full[s, anchors_all[s]] = 1
        mine = [s for s in range(S) if owner_all[s] == rank]
        dcs = [dev_chunk(ns, cs[s], dev, model=models[s], state=True) for s in mine]
        hr = [alloc_hr(n, cs[s], dev, fill=5) for s in mine]
        anc = anc_full[mine] if mine else torch.zeros((0, n), dtype=torch.uint8, device=dev)
        moves = shard.balanced_sr_and_reconstruct(ctx, dcs, models, mine, anc, hr, anchors_all, owner_all,
                                                  list(range(S)), [1] * S, device=dev, transport="peer")
        torch.cuda.synchronize()
        ok = True
        if rank == 0:
            dref = [dev_chunk(ns, cs[s], dev, model=models[s], state=True) for s in range(S)]
            href = [alloc_hr(n, cs[s], dev, fill=5) for s in range(S)]
            ctx.enhance_streams(dref, href, mode=ns.NS_GIVEN_ANCHORS, anchor_in=anc_full, cost=[1] * S, budget=S * n)
            torch.cuda.synchronize()
            for li, s in enumerate(mine):
                for f in range(n):
                    ok &= bool(torch.equal(hr[li][f], href[s][f]))
                ok &= bool(torch.equal(dcs[li].hr_last, dref[s].hr_last))
                ok &= bool(torch.equal(dcs[li].hr_golden, dref[s].hr_golden))
        ctx.close()
        q.put((rank, [tuple(mv) for mv in moves], ok))
    finally:
        dist.destroy_process_group()


def test_peer_transport_two_ranks_one_gpu():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_peer_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    (r0, m0, ok0), (r1, m1, ok1) = res
    assert m0 == m1 and len(m0) >= 3 and all(src == 0 and dst == 1 for _, _, src, dst in m0)
    assert ok0 and ok1
