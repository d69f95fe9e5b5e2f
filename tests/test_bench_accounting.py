"""CPU pins of bench.py's measurement arithmetic:
the algorithmic work the roofline fractions divide by, and the per-shape SR batch
the bench sizes its pool for (mirroring csrc/k_sr.cu sr_batch_jobs)."""
import numpy as np

import bench
import synth


def test_algorithmic_recon_bytes_per_hr_pixel():
    """Reconstruction of a non-anchor inter frame: ref 3 B + write 3 B + residual
    6/s^2 B + MV 0.125/s^2 B per HR pixel (6.68 B at x3); a non-anchor KEY frame:
    write 3 B + LR 3/s^2 B; anchors cost nothing here."""
    cfg = dict(synth.CONFIGS[4])
    S, n, s = 2, 4, cfg["scale"]
    hpx = cfg["h"] * cfg["w"] * s * s
    types = [[synth.NS_KEY, synth.NS_NORMAL, synth.NS_NORMAL, synth.NS_NORMAL]] * S
    ia = np.zeros((S, n), np.uint8)
    ia[:, 1] = 1                                   # one anchor per stream
    _, by = bench.algorithmic(cfg, types, ia, S, n)
    inter = 3 + 3 + 6 / s ** 2 + 0.125 / s ** 2
    key = 3 + 3 / s ** 2
    assert abs(inter - 6.680555) < 1e-5
    assert np.isclose(by["recon"], S * hpx * (2 * inter + key))
    assert np.isclose(by["score"], S * n * cfg["h"] * cfg["w"] * 6)


def test_algorithmic_sr_flops():
    """2 x MACs of the defined convs only: 496,512 FLOP per LR pixel at B8/C32/x3."""
    cfg = dict(synth.CONFIGS[4])
    ia = np.zeros((1, 60), np.uint8)
    ia[0, [0, 12, 24, 36, 48]] = 1
    fl, _ = bench.algorithmic(cfg, [[synth.NS_KEY] + [synth.NS_NORMAL] * 59], ia, 1, 60)
    px = cfg["h"] * cfg["w"] * 5
    assert np.isclose(sum(fl.values()), 496512 * px)
    assert np.isclose(fl["sr_body"], 2 * 9 * 32 * 32 * 2 * 8 * px)


def test_sr_jobs_per_shape():
    """About two waves of the fused residual block on 148 SMs: 16 jobs at 720p,
    49 at 360p, clamped to [16, 64]; a fixed NS_SR_BATCH wins."""
    assert bench.sr_jobs(720, 1280, 148) == 16
    assert bench.sr_jobs(360, 640, 148) == 49
    assert bench.sr_jobs(72, 128, 148) == 64
    assert bench.sr_jobs(2160, 3840, 148) == 16
    assert bench.sr_jobs(360, 640, 148, fixed=16) == 16
