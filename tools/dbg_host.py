import sys, os
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo")); sys.path.insert(0, os.path.join(os.environ.get("GRAFT_REPO_ROOT", "/root/repo"), "tests"))
import numpy as np, torch
import test_gpu_host_path as T
import paper_conf_sigcomm_yeolkjyh22_b200 as ns
c = ns.Context(0, pool_bytes=4 << 30)
shapes = [(64, 32, 2), (64, 32, 2), (48, 24, 3), (64, 32, 2), (48, 24, 3)]
specs = [(2, 16), (1, 16), (1, 32), (2, 16), (1, 32)]
chunks = [T._streams(5100 + 10 * call, shapes, 10, 4) for call in range(2)]
outs = T._run_both(c, chunks, specs, k=3)
for call in range(2):
    d, h = outs["device"][call], outs["host"][call]
    for s in range(5):
        for f in range(10):
            a, b = d["hr"][s][f], h["hr"][s][f]
            if not np.array_equal(a, b):
                diff = np.abs(a.astype(int) - b.astype(int))
                ys, xs = np.nonzero(diff.max(0))
                print("call", call, "stream", s, "frame", f, "anchor", d["ia"][s][f], "type", chunks[call][s].type[f],
                      "n diff px", len(ys), "max", diff.max(), "rows", sorted(set(ys.tolist()))[:8], "cols", sorted(set(xs.tolist()))[:8])
