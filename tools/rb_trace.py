"""Timeline of one CTA of k_resblock (trace build, tools/bin/libneuroscaler_trace.so)."""
import ctypes, os, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sigcomm_yeolkjyh22_b200 as ns
import synth
ns.LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "bin", os.environ.get("NS_TRACE_LIB", "libneuroscaler_trace.so"))
L = ns.lib()
L.ns_trace_read.argtypes = [ctypes.c_void_p, ctypes.c_int]
L.ns_trace_read.restype = ctypes.c_int
ctx = ns.Context(0, pool_bytes=16 << 30)
m = ctx.model(8, 32, 3)
m.set_weights(synth.make_weights(1, 8, 32, 3))
c = synth.make_chunk(5, 1280, 720, 3, 1)
lr = torch.from_numpy(c.lr).cuda()
hr = torch.zeros((16, 3, 2160, 3840), dtype=torch.uint8, device="cuda")
jobs = [(m, lr[0], hr[i]) for i in range(16)]
ctx.sr_anchors(jobs); torch.cuda.synchronize()
L.ns_trace_reset()
# only the first fused block of one batch is traced: regions are overwritten by later launches,
# so run exactly one batch and keep the LAST block's timeline (all blocks behave alike)
ctx.sr_anchors(jobs); torch.cuda.synchronize()
buf = (ctypes.c_ulonglong * (2 * 16384))()
n = L.ns_trace_read(buf, 16384)
a = np.frombuffer(buf, dtype=np.uint64)[:2 * n].reshape(n, 2)
a = a[a[:, 0] != 0]
t = a[:, 0].astype(np.int64); tag = (a[:, 1] >> 32).astype(int); q = (a[:, 1] & 0xffffffff).astype(int)
order = np.argsort(t)
t, tag, q = t[order], tag[order], q[order]
t0 = t[0]
names = {1: "M1 e1z ok A", 2: "M1 e1z ok B", 48: "M2 e2z ok A", 49: "M2 e2z ok B", 50: "M1 hfull ok A", 51: "M1 hfull ok B", 3: "M1 issued A", 4: "M1 issued B", 5: "M2 e1t ok A", 6: "M2 e1t ok B",
         7: "M2 issued A", 8: "M2 issued B", 10: "E1 m1 ok A", 11: "E1 m1 ok B", 12: "E1 arrive A", 13: "E1 arrive B",
         20: "E2 m2 ok A", 21: "E2 m2 ok B", 22: "E2 arrive A", 23: "E2 arrive B", 30: "TMA load A", 31: "TMA load B",
         40: "E1 ld done A", 41: "E1 ld done B", 42: "E1 sts done A", 43: "E1 sts done B", 44: "E1 wait_st A",
         45: "E1 wait_st B", 46: "E1 fence A", 47: "E1 fence B"}
for i in range(len(t)):
    if q[i] < 14 and tag[i] != 30 and tag[i] != 31:
        print(f"{t[i]-t0:8d}  q={q[i]:3d}  {names.get(tag[i], tag[i])}")
# steady state period
# E1 phase durations (tile A), steady state
def col(tg):
    return t[tag == tg][10:60].astype(np.int64)
try:
    m1, ld, sts, fen, arr = col(10), col(40), col(42), col(46), col(12)
    n = min(map(len, (m1, ld, sts, fen, arr)))
    print("E1 A phases (median cycles): ld", int(np.median(ld[:n] - m1[:n])), "zero+arrive+compute+sts", int(np.median(sts[:n] - ld[:n])),
          "fence.proxy", int(np.median(fen[:n] - sts[:n])), "arrive", int(np.median(arr[:n] - fen[:n])))
except Exception as e:
    print("phase summary failed", e)
for tg in (3, 7, 12, 22):
    ts = t[tag == tg]
    if len(ts) > 20:
        d = np.diff(ts[10:60])
        print("tag", names[tg], "median period", int(np.median(d)), "cycles")
