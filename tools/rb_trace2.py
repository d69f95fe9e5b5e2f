"""Steady-state per-stream intervals of the k_resblock timeline (trace build).
Usage: python tools/rb_trace2.py [libname]"""
import ctypes, os, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sigcomm_yeolkjyh22_b200 as ns
import synth
ns.LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "bin", sys.argv[1] if len(sys.argv) > 1 else "libneuroscaler_trace.so")
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
ctx.sr_anchors(jobs); torch.cuda.synchronize()
buf = (ctypes.c_ulonglong * (2 * 16384))()
n = L.ns_trace_read(buf, 16384)
a = np.frombuffer(buf, dtype=np.uint64)[:2 * n].reshape(n, 2)
a = a[a[:, 0] != 0]
t = a[:, 0].astype(np.int64); tag = (a[:, 1] >> 32).astype(int); q = (a[:, 1] & 0xffffffff).astype(int)
def ev(tg):
    d = {}
    for ti, qi in zip(t[tag == tg], q[tag == tg]):
        d[qi] = ti
    return d
E = {tg: ev(tg) for tg in set(tag.tolist())}
qs = range(8, 30)
def med(a_tag, b_tag, dq=0):
    xs = [E[b_tag][x + dq] - E[a_tag][x] for x in qs if x in E.get(a_tag, {}) and x + dq in E.get(b_tag, {})]
    return int(np.median(xs)) if xs else None
for k, nm in ((0, "A"), (1, "B")):
    print(f"tile {nm}: period M1 issue {med(3+k, 3+k, 1)}  M2 issue {med(7+k, 7+k, 1)}")
    print(f"  M1 issued(q) -> E1 m1 ok(q) {med(3+k, 10+k)} | E1 m1 ok -> ld done {med(10+k, 40+k)} | ld done -> sts done {med(40+k, 42+k)}"
          f" | sts -> fence {med(42+k, 46+k)} | fence -> e1t arrive {med(46+k, 12+k)}")
    print(f"  E1 m1 ok(q) -> M1 waits ok(q+1) {med(10+k, 1+k, 1)} -> M1 issued(q+1) {med(1+k, 3+k, 1)}")
    print(f"  E1 arrive(q) -> M2 waits ok(q) {med(12+k, 5+k)} -> M2 issued {med(5+k, 7+k)} -> E2 m2 ok {med(7+k, 20+k)} -> E2 arrive {med(20+k, 22+k)}")
    print(f"  M1 issued(q) -> M2 issued(q) {med(3+k, 7+k)}")
for k, nm in ((0, "A"), (1, "B")):
    print(f"tile {nm}: TMA issued(q) -> M1 waits ok(q) {med(30+k, 1+k)} | E2 arrive(q-2) -> TMA issued(q+3) {med(22+k, 30+k, 5)}"
          f" | E1 e1z? m1ok(q)->M1 waits ok(q+1) {med(10+k, 1+k, 1)} | M1 issued(q) -> TMA issued(q+1) {med(3+k, 30+k, 1)}")
    print(f"  E2 arrive(q) -> M1 waits ok(q+3) {med(22+k, 1+k, 3)} | E2 arrive(q) -> TMA(q+3) {med(22+k, 30+k, 3)}")
