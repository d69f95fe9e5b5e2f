import sys, os
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import numpy as np, torch
import paper_conf_sigcomm_yeolkjyh22_b200 as ns, synth, oracle
shapes = [tuple(int(v) for v in a.split(",")) for a in sys.argv[1:]] or [(1, 16, 2, 32, 16), (1, 32, 3, 48, 16)]
ctx = ns.Context(0, pool_bytes=2 << 30)
for (B, C, s, w, h) in shapes:
    m = ctx.model(B, C, s); blob = synth.make_weights(5, B, C, s); m.set_weights(blob)
    c = synth.make_chunk(7, w, h, s, 1)
    lr = torch.from_numpy(c.lr[0]).cuda(); hr = torch.zeros((3, s*h, s*w), dtype=torch.uint8, device="cuda")
    ctx.sr_anchors([(m, lr, hr)]); torch.cuda.synchronize()
    exp = oracle.sr_forward(c.lr[0], blob, B, C, s)
    d = np.abs(hr.cpu().numpy().astype(int) - exp.astype(int))
    print(B, C, s, w, h, "maxabs", d.max(), "bad px", int((d > 2).sum()), "of", d.size, flush=True)
    if (d > 2).any():
        c_, Y_, X_ = np.nonzero(d > 2)
        print("  rows", sorted(set(Y_.tolist()))[:20], "X range", X_.min(), X_.max(), "X mod s", sorted(set((X_ % s).tolist())),
              "Y mod s", sorted(set((Y_ % s).tolist())), "planes", sorted(set(c_.tolist())))
        print("  first", list(zip(c_[:12].tolist(), Y_[:12].tolist(), X_[:12].tolist())), "vals", hr.cpu().numpy()[c_[:6], Y_[:6], X_[:6]], exp[c_[:6], Y_[:6], X_[:6]])
