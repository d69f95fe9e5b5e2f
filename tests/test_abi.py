"""C-ABI checks that need no GPU: the library builds for sm_100a, loads, and
exports every function include/ns.h declares; ns_model_blob_len agrees with the
oracle's blob layout; argument validation fails without launching anything."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def nslib():
    from paper_conf_sigcomm_yeolkjyh22_b200 import build
    build.build()
    import paper_conf_sigcomm_yeolkjyh22_b200 as ns
    return ns


def header_functions():
    src = open(os.path.join(ROOT, "include", "ns.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ns_[a-z_]+)\s*\(", src)))


def test_exports_every_header_symbol(nslib):
    L = nslib.lib()
    names = header_functions()
    assert len(names) >= 12
    for n in names:
        assert hasattr(L, n), n
    assert sorted(nslib.EXPORTS) == names
    out = subprocess.run(["nm", "-D", "--defined-only", nslib.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (ns_[a-z_]+)$", out, flags=re.M))
    assert set(names) <= exported
    # nothing else with C linkage leaks out
    assert exported == set(names)


def test_sass_is_sm100a_tcgen05(nslib):
    out = subprocess.run(["cuobjdump", "-sass", nslib.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in subprocess.run(["cuobjdump", "-lelf", nslib.LIB_PATH], capture_output=True,
                                       text=True).stdout or "arch = sm_100a" in out
    for mnem in ("UTCHMMA", "UTMALDG", "LDTM"):
        assert mnem in out, mnem


def test_blob_len_matches_oracle(nslib):
    import oracle
    import synth
    for B, C, s in ((4, 16, 2), (8, 32, 3), (1, 32, 4), (3, 16, 3)):
        assert nslib.Model.blob_len(B, C, s) == oracle.blob_len(B, C, s) == synth.blob_len(B, C, s)


def test_invalid_args_no_launch(nslib):
    L = nslib.lib()
    before = nslib.launch_count()
    h = ctypes.c_void_p()
    # no context / bad arguments -> negative status, message set, nothing launched
    assert L.ns_ctx_create(0, 1 << 20, None) == nslib.NS_EINVAL
    assert L.ns_select_anchors(None, None, 0, None, None, None, None, None) == nslib.NS_EINVAL
    assert "NULL" in nslib.last_error()
    assert L.ns_reconstruct_chunk(None, None, 1, None, None, None) == nslib.NS_EINVAL
    assert L.ns_sr_anchors(None, None, 1, None) == nslib.NS_EINVAL
    assert L.ns_select_merge(None, 1, 1, None, None, None, None, None, 0, None, None, None) == nslib.NS_EINVAL
    assert L.ns_model_destroy(None) == nslib.NS_EINVAL
    del h
    assert nslib.launch_count() == before


def test_hybrid_quality_is_table2(nslib):
    """ns_hybrid_quality = Table 2's JPEG column (tests/golden/table2_jpeg_quality.json,
    PAPER.md:668-677): the band edges are inclusive upper bounds."""
    import json
    g = json.load(open(os.path.join(ROOT, "tests", "golden", "table2_jpeg_quality.json")))
    by = {r["fraction"]: r["jpeg"] for r in g["rows"]}

    def band(a, n):  # the paper's bands, evaluated exactly in rationals
        from fractions import Fraction as Fr
        f = Fr(a, n)
        if f <= Fr(5, 100):
            return by["f <= 5%"]
        if f <= Fr(75, 1000):
            return by["5% < f <= 7.5%"]
        if f <= Fr(10, 100):
            return by["7.5% < f <= 10%"]
        return None
    for n in (1, 8, 20, 40, 60, 120, 256):
        for a in range(0, n + 1):
            exp = band(a, n)
            assert nslib.hybrid_quality(a, n) == (-1 if exp is None else exp), (a, n)
    assert nslib.hybrid_quality(5, 60) == 80          # the configs' k = 5 of 60 (8.3%)
    assert nslib.hybrid_quality(3, 60) == 95 and nslib.hybrid_quality(4, 60) == 90
    assert nslib.hybrid_quality(-1, 60) == -1 and nslib.hybrid_quality(1, 0) == -1
