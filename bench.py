#!/usr/bin/env python3
"""bench.py -- NeuroScaler enhancement hot path on B200: enhanced 4K frames/s.

A step = one chunk (60-frame GOP) of every stream on this GPU through the whole
hot path (ns_enhance_streams: score -> Alg. 1 selection -> SR DNN on anchors ->
reuse reconstruction -> state -> stats).  Default workload = BASELINE.json
configs[3] "c4": 64 concurrent 720p->4K x3 streams on one B200, NAS "high"
model (8 blocks, 32 channels), 8% anchors (k = 5 of 60), one content-aware
model per stream.  N GPUs (torchrun) = N independent shards of 64 streams
(weak scaling, no collective on the hot path; NCCL only gathers stats after
timing).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config 4]
  python bench.py --impl reference ...   # the CPU oracle on a bounded sample
"""
from __future__ import annotations

import argparse
import dataclasses
import json
import os
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

METRIC = "enhanced 4K frames/s per B200 & 8×B200; anchor-SR tensor util; reuse HBM GB/s"
UNIT = "4K frames/s"


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return dict(hbm=float(d["hbm_gbs"]), bf16=float(d["bf16_tflops"]),
                    bf16_sus=float(d.get("bf16_tflops_sustained", d["bf16_tflops"])), src="measured")
    return dict(hbm=6650.0, bf16=1590.0, bf16_sus=1400.0, src="fallback (B200_PROFILING.md)")


# ---------------------------------------------------------------- workload
def cfg_of(args):
    c = dict(synth.CONFIGS[args.config])
    c["streams"] = args.streams or c.get("streams", 1)
    return c


INTERPS = {"bilinear": 0, "regular": 1, "smooth": 2, "sharp": 3, "switchable": 4}


def workload_config(cfg, world, select="topk", fmt="444", interp="bilinear"):
    """The `config` object both arms print (same workload, same keys)."""
    S, s, w, h = cfg["streams"], cfg["scale"], cfg["w"], cfg["h"]
    sel = ("top-k per stream" if select == "topk" else
           f"global budget k*S*N = {cfg['k'] * S * world} anchors over all GPUs' streams (§5.2, NEXT-1)")
    fm = "" if fmt == "444" else ", YUV 4:2:0 (NEXT-2)"
    if interp != "bilinear":
        fm += f", VP9 8-tap MC ({interp}, NEXT-2)"
    return {"workload": f"{cfg['name']}: {S} concurrent {w}x{h}->{s * w}x{s * h} x{s} streams per GPU, "
                        f"B{cfg['n_blocks']}/C{cfg['n_ch']}, n={cfg['n']}, k={cfg['k']} ({sel}){fm}",
            "streams_per_gpu": S, "frames_per_step_per_gpu": S * cfg["n"], "parallelism": f"streams x{world}",
            "select": select, "format": fmt, "interp": interp}


def _gen(a):
    seed, w, h, s, n, alt = a[:6]
    mk = synth.make_chunk_i420 if len(a) > 6 and a[6] == "i420" else synth.make_chunk
    return mk(seed, w, h, s, n, types=synth.default_types(n, alt), interp=a[7] if len(a) > 7 else 0)


def gen_pool(cfg, n_distinct, rank, fmt="444", interp=0):
    seeds = [1000 * 4 + rank * 100000 + i for i in range(n_distinct)]
    args = [(sd, cfg["w"], cfg["h"], cfg["scale"], cfg["n"], cfg["altref_every"], fmt, interp) for sd in seeds]
    procs = min(len(args), max(1, (os.cpu_count() or 1)))
    if procs > 1:
        import multiprocessing as mp
        with mp.get_context("fork").Pool(procs) as pool:
            return pool.map(_gen, args)
    return [_gen(a) for a in args]


# ---------------------------------------------------------------- clocks
class Clocks:
    """nvidia-smi sampling of the SM clock and throttle reasons.  The sampler is
    started before the warm-up (its start-up -- process launch and NVML init --
    stalls the driver for milliseconds and must not land in a short timed
    region); every line is stamped on arrival and only the samples taken
    during [begin(), end()] (plus the first one after, which covers the region's
    last 200 ms) are kept."""
    FIELDS = "clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown," \
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap"

    def __init__(self, gpu_index):
        self.idx = gpu_index
        self.p = None
        self.lines = []
        self.t0 = self.t1 = None

    def start(self):
        import threading
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                                       "-i", str(self.idx), "-lms", "200"], stdout=subprocess.PIPE,
                                      stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None
            return

        def reader():
            for line in self.p.stdout:
                self.lines.append((time.time(), line))
        self.th = threading.Thread(target=reader, daemon=True)
        self.th.start()
        deadline = time.time() + 5.0        # settled once the first sample is out
        while time.time() < deadline and not self.lines:
            time.sleep(0.02)

    def begin(self):
        self.t0 = time.time()

    def end(self):
        self.t1 = time.time()
        if self.p:   # wait for one sample after the region
            deadline = self.t1 + 1.0
            while time.time() < deadline and not any(t > self.t1 for t, _ in self.lines):
                time.sleep(0.02)

    def stop(self):
        if not self.p:
            return None
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.th.join(timeout=5)
        t0 = self.t0 if self.t0 is not None else 0.0
        t1 = self.t1 if self.t1 is not None else float("inf")
        inside = [ln for t, ln in self.lines if t0 <= t <= t1]
        after = [ln for t, ln in self.lines if t > t1][:1]
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in inside + after:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) < 6:
                continue
            try:
                sm.append(float(parts[0]))
                mx = float(parts[1])
            except ValueError:
                continue
            for nm, v in zip(names, parts[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return None
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": len(sm)}


# ---------------------------------------------------------------- CPU oracle
def cpu_model():
    """The host CPU the oracle ran on (lscpu's "Model name", from /proc/cpuinfo)."""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return f"{line.split(':', 1)[1].strip()} ({os.cpu_count()} logical CPUs)"
    except OSError:
        pass
    return None


def cpu_sample(cfg, chunk, blob):
    """Times the oracle as it stands on a bounded sample of one stream-chunk and
    converts to the metric: chunk time = score+select (whole chunk) + k x SR
    frame (timed on a row strip, scaled by pixels) + (n-k) x reconstruction of a
    non-anchor frame (timed on 2 frames)."""
    import oracle
    B, C, s, n, k = cfg["n_blocks"], cfg["n_ch"], cfg["scale"], cfg["n"], cfg["k"]
    h, w = chunk.h, chunk.w
    t0 = time.perf_counter()
    sc = oracle.score(chunk.res)
    oracle.select_topk(list(chunk.type), [int(v) for v in sc], k)
    t_sel = time.perf_counter() - t0
    rows = min(h, 48)
    t0 = time.perf_counter()
    oracle.sr_forward(np.ascontiguousarray(chunk.lr[0][:, :rows]), blob, B, C, s)
    t_sr = (time.perf_counter() - t0) * h / rows
    sub = synth.Chunk(w=w, h=h, scale=s, lr=chunk.lr[:3], res=chunk.res[:3], mv=chunk.mv[:3],
                      type=chunk.type[:3].copy(), res_size=chunk.res_size[:3], interp=getattr(chunk, "interp", 0))
    hr = np.zeros((3, 3, s * h, s * w), np.uint8)
    t0 = time.perf_counter()
    oracle.reconstruct(sub, [1, 0, 0], hr)
    t_rec = (time.perf_counter() - t0) / 2
    t_chunk = t_sel + k * t_sr + (n - k) * t_rec
    threads = int(os.environ.get("OMP_NUM_THREADS", os.cpu_count() or 1))
    return dict(value=n / t_chunk, unit=UNIT, cores=threads, kind="oracle", cpu=cpu_model(),
                sample=f"1 stream-chunk of {cfg['name']} ({w}x{h}->x{s}, n={n}, k={k}): score+select on the full "
                       f"chunk ({t_sel:.2f}s), SR on a {w}x{rows} LR strip scaled by pixels ({t_sr:.1f}s/frame, fp64 "
                       f"OpenMP), reconstruction of 2 non-anchor frames ({t_rec:.2f}s/frame, 1 thread)",
                seconds=dict(select=t_sel, sr_frame=t_sr, recon_frame=t_rec))


def run_reference(args):
    """--impl reference: the CPU oracle, as it stands, on this arm's workload."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    # rank 0 alone runs the oracle, on all host cores (torchrun sets OMP_NUM_THREADS=1
    # per rank; nothing has initialised OpenMP in this process yet)
    os.environ["OMP_NUM_THREADS"] = str(os.cpu_count() or 1)
    cfg = cfg_of(args)
    if cfg["w"] is None:  # c5: the sample is one 720p->4K stream-chunk of the mixed fleet
        cfg.update(w=1280, h=720)
    chunk = _gen((4000, cfg["w"], cfg["h"], cfg["scale"], cfg["n"], cfg["altref_every"], "444",
                  INTERPS[args.interp]))
    blob = synth.make_weights(4000, cfg["n_blocks"], cfg["n_ch"], cfg["scale"])
    vals = []
    for i in range(args.warmup + args.steps):
        r = cpu_sample(cfg, chunk, blob)
        if i >= args.warmup:
            vals.append(r["value"])
    v = float(np.mean(vals))
    ms = 1000.0 * cfg["n"] / v
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": dict(workload_config(cfg, args.gpus, interp=args.interp), sample="one stream-chunk of the workload per step "
                                                                    "(see cpu_baseline.sample), scaled to frames/s"),
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": r["cores"], "kind": "oracle", "sample": r["sample"],
                             "cpu": r["cpu"]},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- GPU arm
def algorithmic(cfg, types, ia, S, n, fmt="444"):
    """Algorithmic FLOPs / bytes per kernel family over one step (DESIGN.md
    "Roofline"): the defined convs only; reconstruct = ref 3 B + write 3 B +
    residual 6/s^2 B + MV 0.125/s^2 B per HR pixel of a non-anchor inter frame,
    LR 3/s^2 B + write 3 B for a non-anchor KEY frame."""
    B, C, s, h, w = cfg["n_blocks"], cfg["n_ch"], cfg["scale"], cfg["h"], cfg["w"]
    px, hpx = h * w, h * w * s * s
    pl = 1.5 if fmt == "i420" else 3.0   # planes' worth of samples per pixel (4:2:0: Y + U/4 + V/4)
    anchors = int(ia.sum())
    conv = lambda cin, cout: 2.0 * 9 * cin * cout
    # sr_up = the composed tail o shuffle o upsampler kernel: algorithmic FLOPs are
    # those of the two DEFINED convs (upsampler + HR tail); sr_tail = the exact
    # frame-border fix-up (CUDA cores, no tensor roofline).
    fl = {"sr_head": anchors * px * conv(3, C), "sr_body": anchors * px * conv(C, C) * 2 * B,
          "sr_end": anchors * px * conv(C, C),
          "sr_up": anchors * px * conv(C, s * s * C) + anchors * hpx * conv(C, 3)}
    rec_bytes = 0.0
    for si in range(S):
        for f in range(n):
            if ia[si, f]:
                continue
            if types[si][f] == synth.NS_KEY:
                rec_bytes += hpx * pl + px * pl
            else:
                rec_bytes += hpx * 2 * pl + px * 2 * pl + px * 8 / 64.0
    by = {"recon": rec_bytes, "score": S * n * px * 2 * pl, "state": S * 2 * 2 * hpx * pl,
          "sr_prep": anchors * px * (pl + 32)}
    return fl, by


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--streams", type=int, default=0)
    ap.add_argument("--distinct", type=int, default=8, help="distinct generated streams (replicated on device)")
    ap.add_argument("--e2e-steps", type=int, default=4)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--sr-batch", type=int, default=int(os.environ.get("NS_SR_BATCH", "0")),
                    help="anchors per SR batch (pool sizing; the library reads NS_SR_BATCH); 0 = per frame shape")
    ap.add_argument("--balance", action="store_true",
                    help="with --select global: anchor-level load balancing across GPUs (shard.plan_anchor_moves; "
                         "LR out / HR back point-to-point), then ns_sr_anchors + ns_reconstruct_chunk")
    ap.add_argument("--select", default="topk", choices=["topk", "global"],
                    help="global: §5.2 selection across all GPUs' streams (per-GPU gains, NCCL all_gather, "
                         "ns_select_merge, NS_GIVEN_ANCHORS) inside the timed step")
    ap.add_argument("--ring", type=int, default=3, help="config 5: HR frames per stream (ring)")
    ap.add_argument("--format", default="444", choices=["444", "i420"],
                    help="frame format of the streams (i420: YUV 4:2:0, NEXT-2)")
    ap.add_argument("--transport", default="nccl", choices=["nccl", "peer"],
                    help="--balance: moved anchors by NCCL point-to-point copies, or read/written in place by the "
                         "importing GPU's SR kernels through CUDA IPC peer mappings")
    ap.add_argument("--interp", default="bilinear", choices=list(INTERPS),
                    help="the streams' sub-pel MC: bilinear (Z14) or VP9 8-tap (NEXT-2, R13)")
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend for N > 1 (gloo + NS_BENCH_SHARE_GPU=1: N ranks on one GPU)")
    ap.add_argument("--encode", action="store_true",
                    help="after timing: hybrid-encode one step's SR anchors (ns_encode_anchors, §6.1) and report "
                         "anchors/s and bytes per anchor")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    if args.config == 5:
        return run_c5(args)

    import torch
    import torch.distributed as dist
    import paper_conf_sigcomm_yeolkjyh22_b200 as ns
    from paper_conf_sigcomm_yeolkjyh22_b200 import shard

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    local = gpu_of(local)
    if world > 1:
        init_dist(args, local)
    torch.cuda.set_device(local)
    dev = torch.device(f"cuda:{local}")
    cfg = cfg_of(args)
    S, n, k, s = cfg["streams"], cfg["n"], cfg["k"], cfg["scale"]
    B, C, h, w = cfg["n_blocks"], cfg["n_ch"], cfg["h"], cfg["w"]
    H, W = s * h, s * w
    P = min(args.distinct, S)

    t_gen = time.time()
    i420 = args.format == "i420"
    interp_c = INTERPS[args.interp]
    pool = gen_pool(cfg, P, rank, args.format, interp_c)
    t_gen = time.time() - t_gen

    host_pool = ns.Context.host_pool_bytes(w, h, n, k, S) if args.e2e_steps > 0 else 0
    # two SR arenas: batches alternate between two streams (ns_api.cu run_sr_group)
    nb = sr_jobs(h, w, torch.cuda.get_device_properties(dev).multi_processor_count, args.sr_batch)
    ctx = ns.Context(local, pool_bytes=int((2.4 * ns_arena_gb(cfg, nb, args.format) + 2) * (1 << 30)) +
                     host_pool)
    # per-stream content-aware models: distinct weights per stream
    models = []
    for si in range(S):
        m = ctx.model(B, C, s)
        m.set_weights(synth.make_weights(4000 + rank * 100000 + si, B, C, s))
        models.append(m)
    # device inputs: P generated chunks, copied to S distinct device buffers
    LRF = (h * w * 3 // 2,) if i420 else (3, h, w)      # one LR / residual frame
    HRF = (H * W * 3 // 2,) if i420 else (3, H, W)      # one HR frame
    lr_d = torch.empty((S, n) + LRF, dtype=torch.uint8, device=dev)
    res_d = torch.empty((S, n) + LRF, dtype=torch.int16, device=dev)
    mv_d = torch.empty((S, n, h // 8, w // 8, 8), dtype=torch.uint8, device=dev)
    ty_d = torch.empty((S, n), dtype=torch.uint8, device=dev)
    for si in range(P):
        c = pool[si]
        lr_d[si].copy_(torch.from_numpy(c.lr))
        res_d[si].copy_(torch.from_numpy(c.res))
        mv_d[si].copy_(torch.from_numpy(np.ascontiguousarray(c.mv).view(np.uint8).reshape(n, h // 8, w // 8, 8)))
        ty_d[si].copy_(torch.from_numpy(c.type))
    for si in range(P, S):
        lr_d[si].copy_(lr_d[si % P]); res_d[si].copy_(res_d[si % P])
        mv_d[si].copy_(mv_d[si % P]); ty_d[si].copy_(ty_d[si % P])
    hr = torch.empty((S, n) + HRF, dtype=torch.uint8, device=dev)
    state = torch.zeros((S, 2) + HRF, dtype=torch.uint8, device=dev)
    fmt_c = ns.NS_FMT_I420 if i420 else ns.NS_FMT_444
    chunks = [ns.DeviceChunk(w=w, h=h, scale=s, lr=lr_d[si], res=res_d[si], mv=mv_d[si], type=ty_d[si],
                             model=models[si], hr_last=state[si, 0], hr_golden=state[si, 1], format=fmt_c,
                             interp=interp_c)
              for si in range(S)]
    hr_out = [[hr[si, f] for f in range(n)] for si in range(S)]
    ia = torch.zeros((S, n), dtype=torch.uint8, device=dev)
    stats = torch.zeros((S, 8), dtype=torch.float64, device=dev)
    stream = torch.cuda.current_stream(dev)

    sids = [rank * S + si for si in range(S)]
    cost = [1] * S                    # one resolution and model size: equal T_DNN per anchor
    budget = k * S * world            # the same anchor count as top-k, placed globally

    models_all = {rank * S + si: models[si] for si in range(S)}
    if args.balance:  # every GPU keeps every stream's model (weights are small) to serve moved anchors
        for r in range(world):
            if r == rank:
                continue
            for si in range(S):
                m = ctx.model(B, C, s)
                m.set_weights(synth.make_weights(4000 + r * 100000 + si, B, C, s))
                models_all[r * S + si] = m

    # the global selection's per-stream rows, built once (no host->device copy or
    # host synchronisation inside a step)
    sid_d = torch.tensor(sids, dtype=torch.int32, device=dev)
    cost_d = torch.tensor(cost, dtype=torch.int64, device=dev)
    shape_d = torch.tensor([[w, h, s]] * S, dtype=torch.int32, device=dev)
    counts = shard.row_counts(S, dev) if args.select == "global" else None

    def step():
        if args.select == "global" and args.balance:
            anc, _, allr = shard.select_global_across_ranks(ctx, chunks, sid_d, cost_d, budget, stream=stream,
                                                            return_all=True, shape=shape_d, counts=counts)
            anc_h = allr["anchor"].cpu().numpy()
            sid_h = allr["sid"].cpu().tolist()
            anchors_all = [[int(f) for f in np.nonzero(anc_h[i])[0]] for i in range(len(sid_h))]
            shard.balanced_sr_and_reconstruct(ctx, chunks, models_all, sids, anc, hr_out, anchors_all,
                                              [x // S for x in sid_h], sid_h, allr["cost"].cpu().tolist(),
                                              shape_all=allr["shape"].cpu().tolist(), transport=args.transport)
            ia.copy_(anc)
        elif args.select == "global":
            anc, _ = shard.select_global_across_ranks(ctx, chunks, sid_d, cost_d, budget, stream=stream,
                                                      shape=shape_d, counts=counts)
            ctx.enhance_streams(chunks, hr_out, is_anchor_out=ia, stats=stats, stream=stream,
                                mode=ns.NS_GIVEN_ANCHORS, anchor_in=anc, cost=cost, budget=budget)
        else:
            ctx.enhance_streams(chunks, hr_out, is_anchor_out=ia, stats=stats, k=k, stream=stream)

    clocks = Clocks(int(os.environ.get("CUDA_VISIBLE_DEVICES", str(local)).split(",")[local])
                    if os.environ.get("CUDA_VISIBLE_DEVICES") else local)
    clocks.start()
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    ns.launch_count(reset=True)
    prof_on = os.environ.get("NS_BENCH_NOPROF") != "1"
    ns.profile_enable(prof_on)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev_steps = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    torch.cuda.synchronize(dev)
    clocks.begin()
    e0.record(stream)
    host_t = []
    for i in range(args.steps):
        th0 = time.perf_counter()
        step()
        ev_steps[i].record(stream)
        host_t.append((time.perf_counter() - th0) * 1000.0)
    e1.record(stream)      # before any host work: a short step list may already be done on the GPU
    # host time to enqueue one step: the first call after the synchronize is pure
    # enqueue work (later ones may wait for a staging slot the GPU still reads)
    host_ms = {"first": host_t[0], "median": float(np.median(host_t))}
    torch.cuda.synchronize(dev)
    clocks.end()
    ns.profile_enable(False)
    launches = ns.launch_count()
    ms = e0.elapsed_time(e1)
    step_ms = [e0.elapsed_time(ev_steps[0])] + [ev_steps[i - 1].elapsed_time(ev_steps[i]) for i in range(1, args.steps)]
    clk = clocks.stop()
    prof = ns.profile_read()
    ms = shard.max_over_ranks(ms)      # job time = the slowest rank (device-timed)
    frames = world * S * n * args.steps
    value = frames / (ms / 1000.0)

    # stats gather (the only collective; off the timed region)
    st = shard.gather_stats(stats.clone()).cpu().numpy()
    ia_np = ia.cpu().numpy()
    types = [pool[si % P].type for si in range(S)]

    # rooflines from the live per-family event timing
    pk = peaks()
    fl, by = algorithmic(cfg, types, ia_np, S, n, args.format)
    rl = {}
    busy = prof.pop("any", None)   # union over all families: device time with library work running
    for fam, (nl, ng, tms) in prof.items():
        if nl == 0 or tms <= 0:
            continue
        tot = tms / args.steps
        ent = {"launches_per_step": nl / args.steps, "ms_per_step": tot, "share": tms / ms if world == 1 else None}
        if fam in fl:
            a = fl[fam] / (tot / 1000.0) / 1e12
            ent.update(bound="tensor", achieved=a, unit="TFLOP/s", peak=pk["bf16_sus"], frac=a / pk["bf16_sus"])
            if fam == "sr_up":
                # the composed upsampler o shuffle o tail (one 5x5 conv at LR) executes fewer FLOPs than the
                # two defined convs: its tensor utilisation is the executed work; the algorithmic rate is kept
                # beside it (> 1 of peak by construction, not a utilisation)
                ex = int(ia.sum()) * cfg["h"] * cfg["w"] * 2.0 * 25 * C * 3 * s * s
                e_tf = ex / (tot / 1000.0) / 1e12
                ent.update(achieved=e_tf, frac=e_tf / pk["bf16_sus"], work="executed FLOPs of the composed 5x5 conv",
                           algorithmic_tflops=a, algorithmic_frac=a / pk["bf16_sus"])
        elif fam in by:
            a = by[fam] / (tot / 1000.0) / 1e9
            ent.update(bound="hbm", achieved=a, unit="GB/s", peak=pk["hbm"], frac=a / pk["hbm"])
        rl[fam] = ent
    sr_fams = [f for f in ("sr_prep", "sr_head", "sr_body", "sr_end", "sr_up", "sr_tail") if f in rl]
    sr_ms = sum(rl[f]["ms_per_step"] for f in sr_fams)
    sr_tf = sum(fl.values()) / (sr_ms / 1000.0) / 1e12 if sr_ms else 0.0
    dom = max((f for f in rl if "bound" in rl[f]), key=lambda f: rl[f]["ms_per_step"], default=None)
    roofline = None   # (NS_BENCH_NOPROF=1, a diagnostic run: no per-family timing)
    if dom is not None:
        d = rl[dom]
        traffic = None
        tkey = dom
        per_launch = (fl.get(dom) or by.get(dom)) / max(1, d["launches_per_step"])
        if dom == "recon" and args.interp != "bilinear":
            # 8-tap streams step in k_recon8, one working launch per frame step (the
            # bilinear kernel's launches of the same family return at once)
            tkey, per_launch = "recon8", by[dom] / n
        tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
        if os.path.exists(tp):
            traffic = json.load(open(tp)).get(tkey)
        roofline = {"bound": d["bound"], "achieved": d["achieved"], "peak": d["peak"], "unit": d["unit"],
                    "frac": d["frac"], "traffic": traffic, "kernel": "k_recon8" if tkey == "recon8" else dom,
                    "per_launch_algorithmic": per_launch,
                    "peak_source": f"{pk['src']} ({'bf16 sustained' if d['bound'] == 'tensor' else 'HBM copy'})"}

    # e2e: the public host-input call (ns_enhance_streams_host): every step the
    # library uploads each stream's res/mv/type from pinned host memory (stream
    # groups overlapped with compute on its copy stream) and gathers the
    # anchors' LR frames; then the step's result (stats, anchor map) is read back.
    e2e = None
    if args.e2e_steps > 0:
        hpool = [ns.DeviceChunk.pinned_from_numpy(c.lr, c.res, c.mv, c.type, w, h, s, format=fmt_c, interp=interp_c)
                 for c in pool]
        hchunks = []
        for si in range(S):
            hc = dataclasses.replace(hpool[si % P], model=models[si], hr_last=state[si, 0], hr_golden=state[si, 1])
            hchunks.append(hc)
        st_h = torch.empty((S, 8), dtype=torch.float64).pin_memory()
        ia_h = torch.empty((S, n), dtype=torch.uint8).pin_memory()
        d2h = st_h.numel() * 8 + ia_h.numel()
        moved = [0]

        def e2e_step():
            moved[0] = ctx.enhance_streams_host(hchunks, hr_out, is_anchor_out=ia, stats=stats, k=k, stream=stream)
            st_h.copy_(stats, non_blocking=True)
            ia_h.copy_(ia, non_blocking=True)

        e2e_step()
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
        q0, q1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        q0.record(stream)
        for _ in range(args.e2e_steps):
            e2e_step()
        q1.record(stream)
        torch.cuda.synchronize(dev)
        ems = shard.max_over_ranks(q0.elapsed_time(q1))
        e2e = {"value": world * S * n * args.e2e_steps / (ems / 1000.0), "unit": UNIT, "h2d_bytes_per_step": moved[0],
               "d2h_bytes_per_step": d2h, "steps": args.e2e_steps,
               "api": "ns_enhance_streams_host (C ABI, pinned host inputs)", "select": "topk",
               "note": "per step: H2D of every stream's residual+MV+type (uploaded in stream groups on the library's "
                       "copy stream, overlapped with compute) and of the anchors' LR frames (gathered after "
                       "selection; non-anchor LR is read only for intra blocks, in place); D2H of the per-stream "
                       "stats and anchor map; HR frames stay in HBM for the downstream encoder"}

    # --encode: the whole pipeline to the paper's output (§6.1 hybrid stream):
    # host inputs in, enhance, anchor map back, JPEG of every SR anchor with its
    # per-frame headers, packages in host memory -- host wall clock per step
    e2e_pkg = None
    if args.encode and args.e2e_steps > 0:
        ctx.encode_anchors(hchunks[:1], ia.cpu().numpy()[:1], hr_out[:1])   # encoder setup
        torch.cuda.synchronize(dev)
        t0 = time.perf_counter()
        pkg_bytes = 0
        for _ in range(args.e2e_steps):
            ctx.enhance_streams_host(hchunks, hr_out, is_anchor_out=ia, stats=stats, k=k, stream=stream)
            ia_host = ia.cpu().numpy()
            pkgs = ctx.encode_anchors(hchunks, ia_host, hr_out)
            pkg_bytes = sum(len(p) for p in pkgs)
        t_pkg = time.perf_counter() - t0
        e2e_pkg = {"value": S * n * args.e2e_steps / t_pkg, "unit": UNIT, "steps": args.e2e_steps,
                   "clock": "host wall (the encoder returns host bitstreams)",
                   "h2d_bytes_per_step": moved[0], "d2h_bytes_per_step": pkg_bytes + ia_host.nbytes,
                   "api": "ns_enhance_streams_host + ns_encode_anchors"}

    hybrid = None
    if args.encode:  # §6.1 hybrid encoding of the last step's anchors (off the timed hot path)
        ia_host = ia.cpu().numpy()
        ctx.encode_anchors(chunks[:1], ia_host[:1], hr_out[:1])          # encoder setup, warm-up
        torch.cuda.synchronize(dev)
        t0 = time.perf_counter()
        pkgs = ctx.encode_anchors(chunks, ia_host, hr_out)
        t_enc = time.perf_counter() - t0
        na = int(ia_host.sum())
        hybrid = {"anchors": na, "seconds": t_enc, "anchors_per_s": na / t_enc,
                  "mean_anchor_bytes": (sum(len(p) for p in pkgs) - 16 * S * n) / max(na, 1),
                  "quality": ns.hybrid_quality(k, n), "codec": "JPEG 4:4:4 (nvJPEG), Table 2 quality",
                  "package_bytes": sum(len(p) for p in pkgs)}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline and not i420:
        r = cpu_sample(cfg, pool[0], synth.make_weights(4000, B, C, s))
        cpu = {kk: r[kk] for kk in ("value", "unit", "cores", "kind", "sample", "cpu")}

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True, "scaling": "weak",
                "vs_baseline": None, "dtype": "bf16",
                "data": f"synthetic ({P} generated streams replicated to {S} distinct device buffers per GPU; "
                        f"random-init per-stream weights of the NAS 'high' architecture)",
                "config": dict(workload_config(cfg, world, args.select, args.format, args.interp),
                               balance=bool(args.balance), transport=args.transport if args.balance else None,
                               l2="inputs larger than L2 (~130 GB touched per step)", sr_batch=nb,
                               gen_s=round(t_gen, 1)),
                "roofline": roofline, "rooflines": rl,
                "sr_total": {"ms_per_step": sr_ms, "achieved_tflops": sr_tf, "frac": sr_tf / pk["bf16_sus"],
                             "anchors_per_step": int(ia_np.sum()),
                             "work": "algorithmic FLOPs of the defined convs over the summed SR family times "
                                     "(the families overlap on two SR streams)"},
                "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": int(launches), "clocks": clk,
                "host_enqueue_ms_per_step": host_ms, "step_ms": [round(x, 3) for x in step_ms],
                "e2e_package": e2e_pkg,
                "device_busy_ms_per_step": busy[2] / args.steps if busy else None,
                "hybrid_encode": hybrid,
                # real-time check: one n-frame chunk of every stream (n/60 s of
                # 60 fps video) must finish within its own duration
                "realtime": {"chunk_ms": ms / args.steps, "chunk_video_ms": 1000.0 * n / 60.0,
                             "margin_ms": 1000.0 * n / 60.0 - ms / args.steps,
                             "streams_served_realtime": world * S * min(1.0, (1000.0 * n / 60.0) / (ms / args.steps))},
                "quality": ({"anchors": float(st[:, 1].sum()), "frames": float(st[:, 0].sum())} if not args.balance
                            else None)}  # the balanced path (ns_sr_anchors + ns_reconstruct_chunk) computes no stats
        print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.destroy_process_group()


def gpu_of(local_rank):
    """The device of this rank: LOCAL_RANK, or -- NS_BENCH_SHARE_GPU=1, a test of
    the multi-rank path on a one-GPU box -- every rank on device 0."""
    return 0 if os.environ.get("NS_BENCH_SHARE_GPU") == "1" else local_rank


def init_dist(args, device):
    """NCCL over NVLink between GPUs; --backend gloo (CPU collectives) lets
    several ranks share one GPU (NCCL rejects two ranks on one device)."""
    import torch
    import torch.distributed as dist
    if args.backend == "nccl":
        dist.init_process_group("nccl", device_id=torch.device(f"cuda:{device}"))
    else:
        dist.init_process_group("gloo")


# ---------------------------------------------------------------- c5: mixed fleet
K4_PX = 3840 * 2160


def c5_fleet(n_streams):
    """BASELINE configs[4]: 6 content profiles x 2 resolutions,
    half c3-type 720p->4K, half c2-type 360p->1080p (P:120, P:398 mixed
    fleets), all x3, B8/C32, n = 60, k = 5.  Stream i: resolution by i % 2,
    profile by (i // 2) % 6."""
    out = []
    for i in range(n_streams):
        w, h = (1280, 720) if i % 2 == 0 else (640, 360)
        out.append(dict(sid=i, w=w, h=h, profile=(i // 2) % 6))
    return out


def run_c5(args):
    """512 mixed streams LPT-sharded over the ranks (shard.lpt_shard on the
    analytic per-stream cost), one chunk of every stream of this rank per step
    through ns_enhance_streams, HR outputs in rings of --ring frames per stream
    (the whole-chunk table of 512 streams would need ~1 TB).  value = enhanced
    4K-equivalent frames/s (HR pixels / 3840x2160) over all ranks."""
    import torch
    import torch.distributed as dist
    import paper_conf_sigcomm_yeolkjyh22_b200 as ns
    from paper_conf_sigcomm_yeolkjyh22_b200 import shard

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    local = gpu_of(local)
    if world > 1:
        init_dist(args, local)
    torch.cuda.set_device(local)
    dev = torch.device(f"cuda:{local}")
    cfg = cfg_of(args)
    n, k, s, B, C = cfg["n"], cfg["k"], cfg["scale"], cfg["n_blocks"], cfg["n_ch"]
    fleet = c5_fleet(cfg["streams"])
    costs = [shard.stream_cost(x["w"], x["h"], s, n, k, B, C) for x in fleet]
    mine = [fleet[i] for i in shard.lpt_shard(costs, world)[rank]]
    R = args.ring
    # device input pool: P distinct generated chunks per resolution, streams map
    # onto them round-robin (read-only inputs; streams sharing an entry are
    # >= P streams apart in the launch order, far beyond what L2 holds)
    shapes = sorted({(x["w"], x["h"]) for x in mine}, reverse=True)
    P = args.distinct
    t_gen = time.time()
    pool = {}
    for (w, h) in shapes:
        seeds = [5000 + 1000 * (w // 640) + rank * 100000 + i for i in range(P)]
        a = [(sd, w, h, s, n, cfg["altref_every"]) for sd in seeds]
        import multiprocessing as mp
        with mp.get_context("fork").Pool(min(len(a), os.cpu_count() or 1)) as pp:
            pool[(w, h)] = pp.map(_gen, a)
    t_gen = time.time() - t_gen
    dpool = {}
    for (w, h), cs in pool.items():
        dpool[(w, h)] = [ns.DeviceChunk.from_numpy(c.lr, c.res, c.mv, c.type, w, h, s, dev) for c in cs]
    by_shape = {sh: [x for x in mine if (x["w"], x["h"]) == sh] for sh in shapes}
    S = len(mine)
    # pool: SR arenas (two per shape) + the anchor cache (k anchors per stream)
    acache = sum(len(v) * k * 3 * (s * w) * (s * h) for (w, h), v in by_shape.items())
    sms = torch.cuda.get_device_properties(dev).multi_processor_count
    arenas = sum(2.4 * ns_arena_gb(dict(cfg, w=w, h=h), sr_jobs(h, w, sms, args.sr_batch)) for (w, h) in shapes)
    ctx = ns.Context(local, pool_bytes=int((arenas + 2) * (1 << 30)) + acache + (256 << 20))
    chunks, rows, hr_bufs, states = [], [], [], []
    for (w, h) in shapes:
        grp = by_shape[(w, h)]
        if not grp:
            continue
        H, W = s * h, s * w
        ring = torch.empty((len(grp), R, 3, H, W), dtype=torch.uint8, device=dev)
        st = torch.zeros((len(grp), 2, 3, H, W), dtype=torch.uint8, device=dev)
        hr_bufs.append(ring)
        states.append(st)
        for j, x in enumerate(grp):
            m = ctx.model(B, C, s)
            m.set_weights(synth.make_weights(6000 + x["sid"], B, C, s))
            src = dpool[(w, h)][j % P]
            chunks.append(dataclasses.replace(src, model=m, hr_last=st[j, 0], hr_golden=st[j, 1]))
            rows.append([ring[j, f % R] for f in range(n)])
    ia = torch.zeros((S, n), dtype=torch.uint8, device=dev)
    stats = torch.zeros((S, 8), dtype=torch.float64, device=dev)
    stream = torch.cuda.current_stream(dev)

    def step():
        ctx.enhance_streams(chunks, rows, is_anchor_out=ia, stats=stats, k=k, stream=stream)

    clocks = Clocks(local)
    clocks.start()
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    ns.launch_count(reset=True)
    ns.profile_enable(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(dev)
    clocks.begin()
    e0.record(stream)
    for _ in range(args.steps):
        step()
    e1.record(stream)
    torch.cuda.synchronize(dev)
    clocks.end()
    ns.profile_enable(False)
    launches = ns.launch_count()
    ms_local = e0.elapsed_time(e1)
    clk = clocks.stop()
    prof = ns.profile_read()
    prof.pop("any", None)
    ms = shard.max_over_ranks(ms_local)
    px4k_local = sum(n * 9 * x["w"] * x["h"] for x in mine) / K4_PX      # 4K-equivalent frames per step
    tot = torch.tensor([px4k_local, float(S), float(sum(n for _ in mine))], dtype=torch.float64,
                       device=dev if args.backend == "nccl" else "cpu")
    if world > 1:
        dist.all_reduce(tot)
    px4k, S_all, frames = (float(v) for v in tot.cpu().tolist())
    value = px4k * args.steps / (ms / 1000.0)
    step_ms = ms / args.steps
    hr_gb = sum(b.numel() for b in hr_bufs) / 1e9
    if rank == 0:
        pk = peaks()
        rl = {f: {"launches_per_step": nl / args.steps, "ms_per_step": t / args.steps}
              for f, (nl, ng, t) in prof.items() if nl}
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": step_ms, "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": "bf16",
                "data": f"synthetic ({P} generated chunks per resolution per GPU, streams mapped round-robin; "
                        f"random-init per-stream weights of the NAS 'high' architecture)",
                "config": {"workload": f"c5: {int(S_all)} concurrent mixed streams (half 1280x720->3840x2160, half "
                                       f"640x360->1920x1080, x3, 6 content profiles), B{B}/C{C}, n={n}, k={k}, "
                                       f"LPT-sharded over {world} GPU(s), HR rings of {R} frames per stream",
                           "streams_total": int(S_all), "streams_this_gpu": S, "parallelism": f"streams x{world}",
                           "hr_ring": R, "hr_ring_gb_this_gpu": hr_gb, "anchor_cache_gb": acache / 1e9,
                           "l2": "inputs larger than L2", "gen_s": round(t_gen, 1)},
                "frames_per_s": frames * args.steps / (ms / 1000.0),
                "realtime": {"chunk_ms": step_ms, "chunk_video_ms": 1000.0 * n / 60.0,
                             "margin_ms": 1000.0 * n / 60.0 - step_ms,
                             "streams_served_realtime": S_all * min(1.0, (1000.0 * n / 60.0) / step_ms)},
                "rooflines": rl, "peaks": pk, "gpu_launches": int(launches), "clocks": clk, "e2e": None,
                "cpu_baseline": None}
        print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.destroy_process_group()


def sr_jobs(h, w, sms, fixed=None):
    """Anchors per SR batch of one frame shape, as the library picks them
    (csrc/k_sr.cu sr_batch_jobs): about two waves of the fused residual block."""
    if fixed:
        return fixed
    per_job = -(-h // 240) * ((-(-w // 126) + 1) // 2)
    return min(64, max(16, 2 * sms // max(per_job, 1)))


def ns_arena_gb(cfg, nb, fmt="444"):
    """SR arena of one shape (csrc/k_sr.cu sr_arena_bytes): x0 (8 ch) + h0/hb/tb
    (C ch) bf16 + the u8 LR copy + border bands (small)."""
    h, w, C, s = cfg["h"], cfg["w"], cfg["n_ch"], cfg["scale"]
    px = h * w * nb
    return (px * 8 * 2 + 3 * px * C * 2 + px * 3 + nb * (8 * (w + h) * s * (C + 3) * 4) +
            (3 * s * s * px if fmt == "i420" else 0)) / (1 << 30)


if __name__ == "__main__":
    main()
