import time, sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_sigcomm_yeolkjyh22_b200 as ns, synth
ctx = ns.Context(0, pool_bytes=4 << 30)
n = 20
c = synth.make_chunk(5, 1280, 720, 3, n, types=synth.default_types(n, 8))
m = ctx.model(8, 32, 3); m.set_weights(synth.make_weights(5, 8, 32, 3))
dc = ns.DeviceChunk.from_numpy(c.lr, c.res, c.mv, c.type, 1280, 720, 3, "cuda:0", model=m,
     hr_last=torch.zeros((3,2160,3840),dtype=torch.uint8,device="cuda:0"), hr_golden=torch.zeros((3,2160,3840),dtype=torch.uint8,device="cuda:0"))
hr = [torch.zeros((3,2160,3840),dtype=torch.uint8,device="cuda:0") for _ in range(n)]
ia = torch.zeros((1,n),dtype=torch.uint8,device="cuda:0")
ctx.enhance_streams([dc],[hr],is_anchor_out=ia,k=2); torch.cuda.synchronize()
iah = np.zeros((1,n),np.uint8); iah[0,:] = 1
ctx.encode_anchors([dc], iah[:, :2] if False else np.eye(1, n, 0, dtype=np.uint8), [hr], quality=80)
t=time.perf_counter(); pk = ctx.encode_anchors([dc], iah, [hr], quality=80); dt=time.perf_counter()-t
print(f"OPT_HUFF={os.environ.get('NS_JPEG_OPT_HUFFMAN','0')}: {n} 4K anchors in {dt:.3f}s = {n/dt:.1f}/s, {len(pk[0])/n/1e6:.2f} MB each")
