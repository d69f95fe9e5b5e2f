"""Zero-inference anchor selection, written out from the paper -- ORACLE.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  Pure Python, exact
integers, no numpy arithmetic; one function per step of the paper:

  calc_residual        Alg. 1 lines 15-20
  calc_diff_residual   Eq. 1
  update_residual      Alg. 1 lines 21-25
  estimate_gain        Alg. 1 lines 1-14
  select_topk          Fig. 10 steps 1-4 for one stream
  select_global        Fig. 10 step 3-4 merged over streams + the budget
                       equation of §5.2
  select_key           "Key SR" baseline of §3, reading R6
  select_key_uniform   "Key+Uniform SR" baseline of §3, reading R5

Readings where the paper's text is garbled or silent (SURVEY.md §8(c),
restated in DESIGN.md): Z1 (loop counter, variable names), Z2 (CARRY is the
default; FRESH = literal Alg. 1 line 2 per group), Z3 (explicit reset flags),
Z4 (k = n when no reset lies ahead), Z5 (strict '>' => ties go to the lower
frame index; sort key (gain desc, stream asc, frame asc)), Z6 (KEY gain =
+inf, here the sentinel KEY_GAIN), Z7 ('<=' budget, strict prefix).
"""
from __future__ import annotations

KEY, ALTREF, NORMAL = 0, 1, 2
KEY_GAIN = (1 << 63) - 1          # "equal anchor gain" of key frames, Z6
CARRY, FRESH = 0, 1


INVISIBLE, TYPE_MASK = 0x80, 0x7F


def frame_groups(types):
    """Group of every frame: the type byte without the NS_INVISIBLE flag -- an
    invisible ALTREF is still an alternative reference frame (reading
    R12: invisibility changes what is displayed, not selection)."""
    return [int(t) & TYPE_MASK for t in types]


def calc_residual(types, score):
    """Alg. 1 CalcResidual (lines 15-20): running accumulated residual in
    decode order, cleared at KEY frames.  Returns (residuals, reset) where
    reset[f] marks the frames at which the residual resets (Z3)."""
    residual = 0
    residuals, reset = [], []
    for f in range(len(types)):
        if types[f] == KEY:
            residual = 0
        else:
            residual += score[f]
        residuals.append(residual)
        reset.append(types[f] == KEY)
    return residuals, reset


def calc_diff_residual(residuals, reset, i):
    """Eq. 1: dRes(F[i]) = (k - i) * Res[i], k = the closest index > i at which
    the residual resets (a KEY frame or an already-estimated frame), or n --
    the key frame of the next chunk -- if there is none (Z4)."""
    n = len(residuals)
    k = n
    for j in range(i + 1, n):
        if reset[j]:
            k = j
            break
    return (k - i) * residuals[i]


def update_residual(residuals, reset, index):
    """Alg. 1 UpdateResidual (lines 21-25): subtract delta = residuals[index]
    from index forward until the next reset (Z3 replaces the literal
    'residuals[i] == 0' test, equivalent when every non-KEY score >= 1)."""
    delta = residuals[index]
    i = index
    while i < len(residuals):
        if i > index and reset[i]:
            break
        residuals[i] -= delta
        i += 1
    reset[index] = True


def estimate_gain(candidates, residuals, reset):
    """Alg. 1 EstimateGain (lines 1-14) on one group.  candidates: frame
    indices of the group in ascending order; residuals/reset are updated in
    place.  Returns {frame: gain} and the pick order."""
    done = {c: False for c in candidates}
    gain = {}
    order = []
    N = len(candidates)
    while N > 0:                                  # line 3-4 ("N -= 1", Z1)
        N -= 1
        gain_max = None                           # line 5: -inf
        index_max = None
        for i in candidates:                      # line 6
            if not done[i]:                       # line 7
                g = calc_diff_residual(residuals, reset, i)   # line 8, Eq. 1
                if gain_max is None or g > gain_max:          # line 9: strict '>'
                    index_max, gain_max = i, g                # lines 10-11
        done[index_max] = True                    # line 12
        gain[index_max] = gain_max                # line 13
        order.append(index_max)
        update_residual(residuals, reset, index_max)  # line 14
    return gain, order


def stream_gains(types, score, mode=CARRY):
    """Fig. 10 steps 1-2 for one stream: divide into G_key, G_altref, G_normal
     and estimate the gain of every frame.  Returns gain[f]
    (KEY_GAIN for key frames) and, per group, the greedy pick order."""
    types = frame_groups(types)
    n = len(types)
    g_altref = [f for f in range(n) if types[f] == ALTREF]
    g_normal = [f for f in range(n) if types[f] == NORMAL]
    gain = [KEY_GAIN if types[f] == KEY else None for f in range(n)]
    residuals, reset = calc_residual(types, score)
    ga, oa = estimate_gain(g_altref, residuals, reset)
    if mode == FRESH:                             # literal Alg. 1 line 2 per group (Z2)
        residuals, reset = calc_residual(types, score)
    gn, on = estimate_gain(g_normal, residuals, reset)
    for f, g in list(ga.items()) + list(gn.items()):
        gain[f] = g
    return gain, {"altref": oa, "normal": on}


def stream_order(types, gain):
    """Fig. 10 step 3 within one stream: G_key first (ascending), then
    G_altref, then G_normal, each sorted by gain desc, frame asc (Z5)."""
    types = frame_groups(types)
    n = len(types)
    keys = [f for f in range(n) if types[f] == KEY]
    alt = sorted((f for f in range(n) if types[f] == ALTREF), key=lambda f: (-gain[f], f))
    nor = sorted((f for f in range(n) if types[f] == NORMAL), key=lambda f: (-gain[f], f))
    return keys + alt + nor


def select_topk(types, score, k, mode=CARRY):
    """Per-stream top-k: the first k frames of the priority order are anchors.
    Returns (gain[n], rank[n], is_anchor[n]); rank = position in the order."""
    gain, _ = stream_gains(types, score, mode)
    order = stream_order(types, gain)
    rank = [0] * len(types)
    for pos, f in enumerate(order):
        rank[f] = pos
    is_anchor = [1 if rank[f] < k else 0 for f in range(len(types))]
    return gain, rank, is_anchor


def select_global(streams, cost, budget, mode=CARRY):
    """Global anchor-frame selection over all streams (P:178-180 step 3-4 and
    the equation at: the largest N with sum_{i<=N} T_DNN(AF[i]) <=
    T_intv * M; here `budget` = T_intv * M in the same units as cost[stream]).
    streams: list of (types, score).  Order: G_key^global by (stream, frame),
    then G_altref^global, then G_normal^global, each by (gain desc, stream asc,
    frame asc) (Z5, Z6); the selection is the longest prefix within budget (Z7).
    Returns per-stream lists gain, rank (global position), is_anchor."""
    gains = [stream_gains(t, sc, mode)[0] for t, sc in streams]
    entries = {KEY: [], ALTREF: [], NORMAL: []}
    for s, (types, _) in enumerate(streams):
        for f in range(len(types)):
            entries[types[f]].append((s, f))
    order = sorted(entries[KEY])
    for grp in (ALTREF, NORMAL):
        order += sorted(entries[grp], key=lambda e: (-gains[e[0]][e[1]], e[0], e[1]))
    rank = [[0] * len(t) for t, _ in streams]
    is_anchor = [[0] * len(t) for t, _ in streams]
    total = 0
    taking = True
    for pos, (s, f) in enumerate(order):
        rank[s][f] = pos
        if taking and total + cost[s] <= budget:
            total += cost[s]
            is_anchor[s][f] = 1
        else:
            taking = False                        # strict prefix (Z7)
    return gains, rank, is_anchor


def _rank_from_order(n, order, k):
    rank = [0] * n
    for pos, f in enumerate(order):
        rank[f] = pos
    return rank, [1 if rank[f] < k else 0 for f in range(n)]


def select_key(types, k):
    """Key SR ("applying neural super-resolution only to key frames"):
    order = key frames ascending, then every other frame ascending; the anchors
    are the key frames among the first k (reading R6: k = n selects every key
    frame).  gain = KEY_GAIN for key frames, 0 otherwise."""
    types = frame_groups(types)
    n = len(types)
    keys = [f for f in range(n) if types[f] == KEY]
    order = keys + [f for f in range(n) if types[f] != KEY]
    rank, is_anchor = _rank_from_order(n, order, min(k, len(keys)))
    gain = [KEY_GAIN if types[f] == KEY else 0 for f in range(n)]
    return gain, rank, is_anchor


def select_key_uniform(types, k):
    """Key+Uniform SR ("key frames and equally-spaced normal frames"):
    U = {floor(j * n / k) : 0 <= j < k}, the k equally spaced frames of the
    chunk (reading R5); order = key frames ascending, then the frames of U that
    are not key frames ascending, then the rest ascending; anchors = the first k."""
    types = frame_groups(types)
    n = len(types)
    U = set((j * n) // k for j in range(k)) if k > 0 else set()
    keys = [f for f in range(n) if types[f] == KEY]
    uni = [f for f in range(n) if types[f] != KEY and f in U]
    rest = [f for f in range(n) if types[f] != KEY and f not in U]
    rank, is_anchor = _rank_from_order(n, keys + uni + rest, k)
    gain = [KEY_GAIN if types[f] == KEY else 0 for f in range(n)]
    return gain, rank, is_anchor


def select_global_sid(streams, sid, cost, budget, mode=CARRY):
    """Global selection over streams gathered from several GPUs in any order
    (ns_select_merge): the stream key of the merged order is the global stream
    id sid[i] (reading R7), i.e. select_global over the streams sorted by sid.
    Returns per-input-stream lists gain, rank, is_anchor."""
    perm = sorted(range(len(streams)), key=lambda i: sid[i])
    g, r, a = select_global([streams[i] for i in perm], [cost[i] for i in perm], budget, mode)
    out_g, out_r, out_a = [None] * len(streams), [None] * len(streams), [None] * len(streams)
    for pos, i in enumerate(perm):
        out_g[i], out_r[i], out_a[i] = g[pos], r[pos], a[pos]
    return out_g, out_r, out_a


def merge_gathered(types, gains, sid, cost, budget):
    """Fig. 10 steps 3-4 and the budget equation over
    rows gathered from several GPUs (what ns_select_merge computes): types[i],
    gains[i] per gathered stream row i (gains from Alg. 1 on the owning GPU),
    sid[i] its global stream id (reading R7), cost[i] its T_DNN.  Order: key
    entries by (sid, frame), then G_altref, then G_normal, each by (gain desc,
    sid asc, frame asc); anchors = the longest prefix within budget (Z7).
    Returns per-row lists rank, is_anchor."""
    types = [frame_groups(t) for t in types]
    rows = range(len(types))
    order = sorted(((i, f) for i in rows for f in range(len(types[i])) if types[i][f] == KEY),
                   key=lambda e: (sid[e[0]], e[1]))
    for grp in (ALTREF, NORMAL):
        order += sorted(((i, f) for i in rows for f in range(len(types[i])) if types[i][f] == grp),
                        key=lambda e: (-gains[e[0]][e[1]], sid[e[0]], e[1]))
    rank = [[0] * len(t) for t in types]
    is_anchor = [[0] * len(t) for t in types]
    total, taking = 0, True
    for pos, (i, f) in enumerate(order):
        rank[i][f] = pos
        if taking and total + cost[i] <= budget:
            total += cost[i]
            is_anchor[i][f] = 1
        else:
            taking = False
    return rank, is_anchor
