"""Pins for the CPU oracle against what the paper and the mathematics fix (CPU only).

Each test names the SURVEY.md 8(c) row / paper passage it pins.  The oracle is never checked
against itself: expected values are closed forms, brute force (numpy sums written from the
definition in a different form), hand computations (tests/golden/), or invariants.
"""
import math
import os

import numpy as np
import pytest

import fdgen
import oracle
import softcasc

GOLD = os.path.join(os.path.dirname(__file__), "golden")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _golden(name):
    rows = []
    with open(os.path.join(GOLD, name)) as fh:
        for line in fh:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    return rows


def cascade_text(stages, soft=False):
    """stages: list of (T, [ (rects, theta, left, right), ... ]); soft: soft cascade (R8b)"""
    out = ["FDC 1", "window 24 24"] + (["soft"] if soft else []) + [f"stages {len(stages)}"]
    for T, stumps in stages:
        out.append(f"stage {len(stumps)} {float(T)!r}" if math.isfinite(T) else f"stage {len(stumps)} {'inf' if T > 0 else '-inf'}")
        for rects, th, l, r in stumps:
            rs = " ".join(" ".join(str(v) for v in rc) for rc in rects)
            out.append(f"stump {len(rects)} {rs} {np.float32(th).item()!r} {np.float32(l).item()!r} {np.float32(r).item()!r}")
    return "\n".join(out) + "\n"


# ---------------------------------------------------------------- c1: pyramid geometry
@pytest.mark.parametrize("row", [r for r in _golden("pyramid_counts.txt") if r[0][0].isdigit()])
def test_plan_closed_form_totals(row):
    W, H, s, step, nl, tot = int(row[0]), int(row[1]), float(row[2]), int(row[3]), int(row[4]), int(row[5])
    lv = oracle.plan(W, H, 24, s, step)
    assert len(lv) == nl
    assert sum(l[3] for l in lv) == tot
    # closed form written independently: f_k by repeated multiply, floor rule
    f = 1.0
    for k, (fk, wk, hk, nw) in enumerate(lv):
        assert fk == f
        assert wk == math.floor(W / f) and hk == math.floor(H / f)
        assert nw == ((wk - 24) // step + 1) * ((hk - 24) // step + 1)
        f = f * s
    assert math.floor(W / f) < 24 or math.floor(H / f) < 24


def test_plan_per_level_counts():
    for row in _golden("pyramid_counts.txt"):
        if row[0] == "levels":
            W, H, s = int(row[1]), int(row[2]), float(row[3])
            assert [l[3] for l in oracle.plan(W, H, 24, s, 1)] == [int(v) for v in row[4:]]
        elif row[0] == "dims":
            k, wk, hk, nw = (int(v) for v in row[1:])
            lv = oracle.plan(1920, 1080, 24, 1.1, 1)[k]
            assert (lv[1], lv[2], lv[3]) == (wk, hk, nw)


@pytest.mark.parametrize("W,H,s", [(320, 240, 1.25), (640, 480, 1.2), (1920, 1080, 1.1), (3840, 2160, 1.1)])
def test_backprojection_inside_frame(W, H, s):
    # c1/c9 invariant: the last window of every level back-projects inside the frame
    for (f, wk, hk, _n) in oracle.plan(W, H, 24, s, 1):
        x = math.floor((wk - 24) * f + 0.5)
        y = math.floor((hk - 24) * f + 0.5)
        w = math.floor(24 * f + 0.5)
        assert x + w <= W and y + w <= H


def test_plan_rejects_bad_args():
    with pytest.raises(ValueError):
        oracle.plan(20, 240, 24, 1.25, 1)
    with pytest.raises(ValueError):
        oracle.plan(320, 240, 24, 1.0, 1)
    with pytest.raises(ValueError):
        oracle.plan(320, 240, 16, 1.25, 1)


# ---------------------------------------------------------------- c2: scaling
def _resample_naive(img, f, Wk, Hk):
    """Second, differently written bilinear: interpolate along x then y, with exact rationals
    for the Q16 sample position (centre-aligned (x+1/2)f - 1/2, 8-bit weights, clamp)."""
    from fractions import Fraction
    H, W = img.shape
    r = Fraction(int(math.floor(f * 65536 + 0.5)), 65536)
    out = np.zeros((Hk, Wk), np.uint8)
    for y in range(Hk):
        sy = (y + Fraction(1, 2)) * r - Fraction(1, 2)
        y0 = min(math.floor(sy), H - 1)
        wy = math.floor((sy - math.floor(sy)) * 256)
        y1 = min(y0 + 1, H - 1)
        for x in range(Wk):
            sx = (x + Fraction(1, 2)) * r - Fraction(1, 2)
            x0 = min(math.floor(sx), W - 1)
            wx = math.floor((sx - math.floor(sx)) * 256)
            x1 = min(x0 + 1, W - 1)
            top = int(img[y0, x0]) * (256 - wx) + int(img[y0, x1]) * wx
            bot = int(img[y1, x0]) * (256 - wx) + int(img[y1, x1]) * wx
            out[y, x] = (top * (256 - wy) + bot * wy + 32768) >> 16
    return out


def test_resample_level0_identity():
    fr = fdgen.background(1, 7, 320, 240)
    f, wk, hk, _ = oracle.plan(320, 240, 24, 1.25, 1)[0]
    assert f == 1.0 and (wk, hk) == (320, 240)
    np.testing.assert_array_equal(oracle.resample(fr, f, wk, hk), fr)


def test_resample_constant_frame():
    fr = np.full((97, 131), 173, np.uint8)
    for (f, wk, hk, _) in oracle.plan(131, 97, 24, 1.13, 1):
        assert (oracle.resample(fr, f, wk, hk) == 173).all()


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_resample_matches_naive(seed):
    rng = np.random.default_rng(seed)
    fr = rng.integers(0, 256, (53, 61), dtype=np.uint8)
    for (f, wk, hk, _) in oracle.plan(61, 53, 24, 1.17, 1):
        np.testing.assert_array_equal(oracle.resample(fr, f, wk, hk), _resample_naive(fr, f, wk, hk))


def test_resample_linear_ramp():
    # bilinear reproduces a linear ramp: value ~ a*(x+1/2)f - 1/2 ... within 1 grey level
    W, H = 200, 40
    fr = np.tile(np.arange(W, dtype=np.int64), (H, 1)).astype(np.uint8)
    for (f, wk, hk, _) in oracle.plan(W, H, 24, 1.3, 1)[:4]:
        lv = oracle.resample(fr, f, wk, hk).astype(np.float64)
        xs = (np.arange(wk) + 0.5) * f - 0.5
        np.testing.assert_allclose(lv[hk // 2, : wk - 2], xs[: wk - 2], atol=1.01)


# ---------------------------------------------------------------- c3: integral images
@pytest.mark.parametrize("seed", [0, 1])
def test_integral_brute_force_all_rects(seed):
    rng = np.random.default_rng(seed)
    img = rng.integers(0, 256, (9, 11), dtype=np.uint8)
    ii, sq = oracle.integral(img)
    I = img.astype(np.int64)
    for y in range(10):
        for x in range(12):
            assert ii[y, x] == I[:y, :x].sum()
            assert sq[y, x] == (I[:y, :x] ** 2).sum()
    for y in range(9):
        for x in range(11):
            for h in range(1, 10 - y):
                for w in range(1, 12 - x):
                    assert oracle.rect_sum(ii, x, y, w, h) == I[y:y + h, x:x + w].sum()


def test_integral_constant_closed_form():
    c = 201
    img = np.full((30, 41), c, np.uint8)
    ii, sq = oracle.integral(img)
    y, x = np.mgrid[0:31, 0:42]
    np.testing.assert_array_equal(ii, (c * x * y).astype(np.uint32))
    np.testing.assert_array_equal(sq, (c * c * x * y).astype(np.uint64))


def test_integral_total_and_u32_range():
    # worst case 1080p all-255: ii max 255*1920*1080 fits u32; sqii needs u64
    img = np.full((1080, 1920), 255, np.uint8)
    ii, sq = oracle.integral(img)
    assert int(ii[-1, -1]) == 255 * 1920 * 1080 == 528768000
    assert int(sq[-1, -1]) == 255 * 255 * 1920 * 1080 > 2 ** 32


# ---------------------------------------------------------------- c5: variance normalisation
def test_nf_constant_window():
    ii, sq = oracle.integral(np.full((24, 24), 77, np.uint8))
    assert oracle.window_nf(ii, sq, 0, 0) == 1.0


@pytest.mark.parametrize("a,b", [(0, 255), (10, 20), (255, 0), (3, 200)])
def test_nf_two_valued_windows(a, b):
    # half/half and checkerboard with values a,b: v = (288 |a-b|)^2, nf = 288 |a-b|
    half = np.full((24, 24), a, np.uint8)
    half[:, 12:] = b
    chk = np.where((np.add.outer(np.arange(24), np.arange(24)) % 2) == 0, a, b).astype(np.uint8)
    for img in (half, chk):
        ii, sq = oracle.integral(img)
        assert oracle.window_nf(ii, sq, 0, 0) == 288.0 * abs(a - b)


# ---------------------------------------------------------------- c6: features (Table I, Fig. 4)
def test_table1_counts():
    want = {r[0]: int(r[1]) for r in _golden("table1.txt")}
    assert fdgen.table1_counts() == want


def test_families_zero_on_constant_window():
    ii, _ = oracle.integral(np.full((24, 24), 93, np.uint8))
    rng = np.random.default_rng(5)
    counts = fdgen.table1_counts()
    for fam in counts:
        for idx in rng.integers(0, counts[fam], 50):
            assert oracle.feature(ii, 0, 0, fdgen.table1_feature(fam, int(idx))) == 0


def test_fig4_edge_expression_unpadded_integral():
    """Fig. 4: eval = (-1)(r[h0]+r[h1]-r[h2]-r[h3]) + 2(r[h4]+r[h5]-r[h6]-r[h7]) over the
    576-row unpadded 24x24 integral J.  Table I features start at offset >= 1, so the
    paper's corners J[y-1][x-1] ... equal the padded ii[y][x] ...: the oracle must agree."""
    rng = np.random.default_rng(11)
    img = rng.integers(0, 256, (24, 24), dtype=np.uint8)
    J = img.astype(np.int64).cumsum(0).cumsum(1)       # unpadded inclusive integral
    ii, _ = oracle.integral(img)
    counts = fdgen.table1_counts()
    for idx in rng.integers(0, counts["edge"], 200):
        rects = fdgen.table1_feature("edge", int(idx))
        (x0, y0, w0, h0, _), (x1, y1, w1, h1, _) = rects

        def rsum(x, y, w, h):  # r[A] + r[D] - r[B] - r[C] with corners just outside the rect
            return J[y + h - 1, x + w - 1] + J[y - 1, x - 1] - J[y - 1, x + w - 1] - J[y + h - 1, x - 1]
        ev = -1 * rsum(x0, y0, w0, h0) + 2 * rsum(x1, y1, w1, h1)
        assert oracle.feature(ii, 0, 0, rects) == ev
        # and against a direct pixel sum
        direct = -int(img[y0:y0 + h0, x0:x0 + w0].astype(np.int64).sum()) + 2 * int(img[y1:y1 + h1, x1:x1 + w1].astype(np.int64).sum())
        assert ev == direct


# ---------------------------------------------------------------- c7/c8: stump, stages
def _worked_window():
    img = np.zeros((24, 24), np.uint8)
    img[:, 12:] = 255
    return img


def test_worked_example_single_stump():
    g = {r[0]: r[1] for r in _golden("worked_example.txt")}
    img = _worked_window()
    ii, sq = oracle.integral(img)
    whole, half = (1, 1, 22, 22, -1), (1, 1, 11, 22, 2)
    assert oracle.rect_sum(ii, 1, 1, 22, 22) == int(g["R_whole"])
    assert oracle.rect_sum(ii, 1, 1, 11, 22) == int(g["R_half"])
    assert oracle.feature(ii, 0, 0, [whole, half]) == int(g["f"])
    assert oracle.window_nf(ii, sq, 0, 0) == float(g["nf"])
    casc = oracle.Cascade(cascade_text([(-10.0, [([whole, half], -0.5, 0.25, 0.75)])]))
    d, score, near = oracle.eval_window(casc, ii, sq, 0, 0)
    assert g["leaf"] == "left" and score == np.float32(0.25) and d == 1 and near == 0
    # the same stump with theta = -1.0: t = -73440 < f -> right leaf
    casc2 = oracle.Cascade(cascade_text([(-10.0, [([whole, half], -1.0, 0.25, 0.75)])]))
    assert oracle.eval_window(casc2, ii, sq, 0, 0)[1] == np.float32(0.75)


def test_stump_tie_goes_right():
    # constant window: f = 0, nf = 1; theta = 0 -> t = 0, (0 < 0) false -> right leaf (c7)
    ii, sq = oracle.integral(np.full((24, 24), 50, np.uint8))
    casc = oracle.Cascade(cascade_text([(-10.0, [([(1, 1, 4, 4, -1), (1, 1, 2, 4, 2)], 0.0, -1.0, 1.0)])]))
    d, score, near = oracle.eval_window(casc, ii, sq, 0, 0)
    assert score == 1.0 and near & 2


def test_stage_pass_on_equality_and_early_exit():
    ii, sq = oracle.integral(_worked_window())
    st = ([(1, 1, 22, 22, -1), (1, 1, 11, 22, 2)], -0.5, 0.25, 0.75)     # leaf 0.25
    # stage 0 threshold exactly 0.5 = 0.25 + 0.25 -> pass (>=); stage 1 threshold 0.26 > 0.25 -> reject
    casc = oracle.Cascade(cascade_text([(0.5, [st, st]), (0.26, [st]), (-1.0, [st])]))
    d, score, near = oracle.eval_window(casc, ii, sq, 0, 0)
    assert d == 1 and score == np.float32(0.25)


def test_soft_cascade_worked_example():
    """f4 soft cascade (ref [32]; reading R8b) on the c7 worked-example window,
    hand-computed: leaves 0.5 then 0.25 (both 'left', f = -61710 < theta*nf = -36720).
    Hard: stage 2 sum 0.25 < 0.7 -> depth 1, score 0.25.  Soft: running sum 0.5 >= 0.4, then
    0.75 >= 0.7 -> accepted, depth 2, score 0.75.  With T_2 = 0.8: 0.75 < 0.8 -> depth 1, 0.75."""
    ii, sq = oracle.integral(_worked_window())
    edge = [(1, 1, 22, 22, -1), (1, 1, 11, 22, 2)]
    stages = [(0.4, [(edge, -0.5, 0.5, -1.0)]), (0.7, [(edge, -0.5, 0.25, -1.0)])]
    d, score, _ = oracle.eval_window(oracle.Cascade(cascade_text(stages)), ii, sq, 0, 0)
    assert d == 1 and score == np.float32(0.25)
    d, score, _ = oracle.eval_window(oracle.Cascade(cascade_text(stages, soft=True)), ii, sq, 0, 0)
    assert d == 2 and score == np.float32(0.75)
    stages[1] = (0.8, stages[1][1])
    d, score, _ = oracle.eval_window(oracle.Cascade(cascade_text(stages, soft=True)), ii, sq, 0, 0)
    assert d == 1 and score == np.float32(0.75)


def test_soft_cascade_equals_prefix_hard_cascades():
    """R8b pinned against the hard-cascade definition (R8, itself pinned above): the soft running
    sum after stage t is the fp32 sequential sum of the leaves of stumps 1..S_t in order, i.e.
    the score of a ONE-stage hard cascade holding those stumps with T = -inf.  So the soft depth
    of a window is the first t with that prefix score < T_t, and its score is that prefix score
    (the full sum if every stage passes).  Checked on every window of a 160x120 frame."""
    W, H, s = 160, 120, 1.25
    fr, _ = fdgen.frames(2, 5, 1, W, H)
    soft_text = softcasc.soft_from("c2.fdc", 6)
    soft = oracle.Cascade(soft_text)
    d, sc, _ = oracle.detect_depth(soft, fr, 24, s, 1, nthreads=4)
    lines = soft_text.splitlines()
    stage_rows = [i for i, ln in enumerate(lines) if ln.startswith("stage ")]
    T = [float(lines[i].split()[2]) for i in stage_rows]
    prefix_scores = []
    for t in range(len(stage_rows)):
        end = stage_rows[t + 1] if t + 1 < len(stage_rows) else len(lines)
        stumps = [ln for ln in lines[stage_rows[0]:end] if ln.startswith("stump ")]
        hard = "\n".join(["FDC 1", "window 24 24", "stages 1", f"stage {len(stumps)} -inf"] + stumps) + "\n"
        _, ps, _ = oracle.detect_depth(oracle.Cascade(hard), fr, 24, s, 1, nthreads=4)
        prefix_scores.append(ps)
    P = np.stack(prefix_scores)                      # [stages, windows]
    fail = P < np.asarray(T, np.float32)[:, None]
    exp_d = np.where(fail.any(axis=0), fail.argmax(axis=0), len(T))
    exp_sc = P[np.minimum(exp_d, len(T) - 1), np.arange(P.shape[1])]
    assert np.array_equal(d, exp_d.astype(d.dtype))
    assert np.array_equal(sc.view(np.uint32), exp_sc.view(np.uint32))
    # non-trivial: windows stop at several depths and some pass everything
    assert len(np.unique(d)) >= 4
    # a one-stage soft cascade is the hard cascade
    one = "\n".join(lines[:stage_rows[1]]) + "\n"
    one = one.replace("stages 6", "stages 1")
    d1, s1, _ = oracle.detect_depth(oracle.Cascade(one), fr, 24, s, 1, nthreads=4)
    d0, s0, _ = oracle.detect_depth(oracle.Cascade(one.replace("soft\n", "")), fr, 24, s, 1, nthreads=4)
    assert np.array_equal(d1, d0) and np.array_equal(s1.view(np.uint32), s0.view(np.uint32))


def test_all_pass_and_all_reject_cascades():
    W, H, s = 160, 120, 1.25
    fr, _ = fdgen.frames(9, 3, 2, W, H)
    st = ([(1, 1, 10, 10, -1), (1, 1, 5, 10, 2)], 0.1, 0.5, 0.5)
    allpass = oracle.Cascade(cascade_text([(-math.inf, [st, st]), (-1e30, [st])]))
    dets, _ = oracle.detect(allpass, fr, 24, s, 1, nthreads=2)
    tot = sum(l[3] for l in oracle.plan(W, H, 24, s, 1))
    assert len(dets) == 2 * tot
    assert (dets["aux"] == 2).all()
    allrej = oracle.Cascade(cascade_text([(math.inf, [st])]))
    d, sc, nr = oracle.detect_depth(allrej, fr, 24, s, 1)
    assert len(d) == 2 * tot and (d == 0).all() and (sc == 0.5).all()


@pytest.mark.parametrize("min_size,num,den", [(36, 3, 2), (30, 5, 4), (48, 2, 1)])
def test_backprojection_round_half_up(min_size, num, den):
    """c9 ("multiplying the downscaling factor by the normalized dimensions"; reading
    R9: round half up in double).  min_size 36 gives f_0 = 1.5 exactly and min_size 30 gives
    1.25, so wx*f_0 lands exactly on .5 for odd wx (1.5 -> 2, 4.5 -> 5) and for wx = 2 mod 4
    (2.5 -> 3).  Expected values are integer closed forms: floor(wx*num/den + 1/2) =
    (2*wx*num + den) // (2*den); round-half-even or truncation would fail at those windows.
    An all-pass cascade makes every level-0 window a detection."""
    W, H = 160, 100
    fr, _ = fdgen.frames(9, 5, 1, W, H)
    st = ([(1, 1, 10, 10, -1), (1, 1, 5, 10, 2)], 0.1, 0.5, 0.5)
    allpass = oracle.Cascade(cascade_text([(-math.inf, [st])]))
    dets, _ = oracle.detect(allpass, fr, min_size, 1.25, 1)
    lv0 = dets[dets["level"] == 0]
    f0 = oracle.plan(W, H, min_size, 1.25, 1)[0]
    assert f0[0] * den == num and len(lv0) == f0[3]
    for field, src in (("x", "wx"), ("y", "wy")):
        want = (2 * lv0[src].astype(np.int64) * num + den) // (2 * den)
        assert np.array_equal(lv0[field], want), field
    assert (lv0["w"] == (2 * 24 * num + den) // (2 * den)).all() and (lv0["h"] == lv0["w"]).all()
    # the half-way cases are present: odd wx for f = 1.5, wx = 2 mod 4 for f = 1.25
    half = (2 * lv0["wx"].astype(np.int64) * num) % (2 * den) == den
    assert half.any() == (den > 1)
    if den > 1:
        assert (lv0["x"][half] * 2 * den == 2 * lv0["wx"][half] * num + den).all()


def test_stage_near_threshold_flag():
    """c11 (north_star: windows whose score lies within 1e-4 of a stage threshold are counted
    and reported): bit 0 of the near flag is set iff |sum_s - T_s| <= 1e-4 at an evaluated
    stage.  Constant window: f = 0, nf = 1; theta = 100 puts every stump far from its own
    threshold (bit 1 clear); both leaves are 0.5 so the stage sum is exactly 0.5."""
    ii, sq = oracle.integral(np.full((24, 24), 77, np.uint8))
    st = ([(1, 1, 4, 4, -1), (1, 1, 2, 4, 2)], 100.0, 0.5, 0.5)
    for T, depth, flag in ((0.5 + 5e-5, 0, 1),      # just above: reject, flagged
                           (0.5 - 5e-5, 1, 1),      # just below: pass, flagged
                           (0.5 + 2e-4, 0, 0),      # outside the band: reject, not flagged
                           (0.5 - 2e-4, 1, 0)):
        d, score, near = oracle.eval_window(oracle.Cascade(cascade_text([(T, [st])])), ii, sq, 0, 0)
        assert (d, score, near) == (depth, 0.5, flag), T
    # the flag comes from any evaluated stage, not only the rejecting one; an unevaluated
    # stage never sets it
    far, close = (0.5 - 2e-4, [st]), (0.5 - 5e-5, [st])
    assert oracle.eval_window(oracle.Cascade(cascade_text([close, far, (1.0, [st])])), ii, sq, 0, 0)[2] == 1
    assert oracle.eval_window(oracle.Cascade(cascade_text([(1.0, [st]), close])), ii, sq, 0, 0)[2] == 0


def test_filter_binomial_pins():
    """f2 filtering stage (reading R3b): weights sum to 16, so constants are fixed points; the
    binomial kernel reproduces linear functions exactly away from the border; an impulse gives
    the 1-2-1 x 1-2-1 stencil with round-half-up; clamp-to-edge at the border (hand values)."""
    c = np.full((30, 40), 173, np.uint8)
    assert np.array_equal(oracle.filter_binomial(c), c)
    x = np.arange(40)
    ramp = np.tile((3 * x + 7).astype(np.uint8), (30, 1))
    f = oracle.filter_binomial(ramp)
    assert np.array_equal(f[:, 1:-1], ramp[:, 1:-1])
    # left border: (1*7 + 2*7 + 1*10) * 4 / 16 = 7.75 -> (124 + 8) >> 4 = 8; right: 124,124,121 -> 123
    assert (f[:, 0] == 8).all() and (f[:, -1] == ((4 * (124 + 2 * 124 + 121) + 8) >> 4)).all()
    imp = np.zeros((7, 7), np.uint8)
    imp[3, 3] = 255
    want = np.zeros((7, 7), np.uint8)
    want[2:5, 2:5] = [[16, 32, 16], [32, 64, 32], [16, 32, 16]]
    assert np.array_equal(oracle.filter_binomial(imp), want)
    # a cascade with 'filter binomial3' evaluates on filtered levels: a constant frame stays
    # constant, so every window has nf = 1 and the same depth as without the filter
    st = ([(1, 1, 10, 10, -1), (1, 1, 5, 10, 2)], 0.1, 0.5, -0.5)
    text = cascade_text([(0.0, [st])])
    filt = text.replace("window 24 24\n", "window 24 24\nfilter binomial3\n")
    fr = np.full((1, 48, 64), 90, np.uint8)
    a, _, _ = oracle.detect_depth(oracle.Cascade(text), fr, 24, 1.25, 1)
    b, _, _ = oracle.detect_depth(oracle.Cascade(filt), fr, 24, 1.25, 1)
    assert np.array_equal(a, b)
    with pytest.raises(Exception):
        oracle.Cascade(text.replace("window 24 24\n", "window 24 24\nfilter gauss\n"))


def test_c6_cascade_shape():
    """f3 workload: the OpenCV-shaped cascade has the paper's "25 stages ... 2913 weak
    classifiers" and only Table I features (2 or 3 rectangles)."""
    casc = oracle.Cascade.from_file(os.path.join(ROOT, "cascades", "c6.fdc"))
    assert casc.n_stages == 25
    sizes, nrects = [], []
    for line in open(os.path.join(ROOT, "cascades", "c6.fdc")):
        t = line.split()
        if t and t[0] == "stage":
            sizes.append(int(t[1]))
        elif t and t[0] == "stump":
            nrects.append(int(t[1]))
    assert sum(sizes) == 2913 == len(nrects) and set(nrects) <= {2, 3}


def test_depth_histogram_pins():
    """f4 (Fig. 7 analytics): hand example, the all-pass / all-reject cascades, and the
    closed-form per-level window counts of tests/golden/pyramid_counts.txt as row sums."""
    # 25 x 25 frame, scale 1.1: one level of 2 x 2 windows; depths [0, 3, 3, 1] (+ a 200 clamp)
    h = oracle.depth_histogram(np.array([0, 3, 3, 1], np.uint8), 1, 25, 25, 3, 24, 1.1, 1)
    assert h.tolist() == [[1, 1, 0, 2]]
    h = oracle.depth_histogram(np.array([0, 200, 3, 1, 2, 2, 2, 2], np.uint8), 2, 25, 25, 3, 24, 1.1, 1)
    assert h.tolist() == [[1, 1, 4, 2]]
    W, H, s = 160, 120, 1.25
    fr, _ = fdgen.frames(9, 3, 2, W, H)
    st = ([(1, 1, 10, 10, -1), (1, 1, 5, 10, 2)], 0.1, 0.5, 0.5)
    allpass = oracle.Cascade(cascade_text([(-math.inf, [st, st]), (-1e30, [st])]))
    d, _, _ = oracle.detect_depth(allpass, fr, 24, s, 1)
    h = oracle.depth_histogram(d, 2, W, H, 2, 24, s, 1)
    per_level = [2 * l[3] for l in oracle.plan(W, H, 24, s, 1)]
    assert h[:, 2].tolist() == per_level and h[:, :2].sum() == 0
    allrej = oracle.Cascade(cascade_text([(math.inf, [st])]))
    d, _, _ = oracle.detect_depth(allrej, fr, 24, s, 1)
    h = oracle.depth_histogram(d, 2, W, H, 1, 24, s, 1)
    assert h[:, 0].tolist() == per_level and h[:, 1].sum() == 0
    # row sums = the closed-form window counts (golden) for the c1 geometry
    row = [r for r in _golden("pyramid_counts.txt") if r[:4] == ["320", "240", "1.25", "1"]][0]
    fr, _ = fdgen.frames(1, 0, 1, 320, 240)
    casc = oracle.Cascade.from_file(os.path.join(ROOT, "cascades", "c1.fdc"))
    d, _, _ = oracle.detect_depth(casc, fr, 24, 1.25, 1, nthreads=4)
    h = oracle.depth_histogram(d, 1, 320, 240, casc.n_stages, 24, 1.25, 1)
    assert len(h) == int(row[4]) and h.sum() == int(row[5])
    assert h.sum(axis=0)[casc.n_stages] == (d == casc.n_stages).sum()


def test_detect_matches_depth_maps_and_order():
    fr, _ = fdgen.frames(1, 0, 2, 320, 240)
    casc = oracle.Cascade.from_file(os.path.join(ROOT, "cascades", "c1.fdc"))
    dets, _ = oracle.detect(casc, fr, 24, 1.25, 1, nthreads=4)
    d, sc, _ = oracle.detect_depth(casc, fr, 24, 1.25, 1, nthreads=4)
    assert (d == casc.n_stages).sum() == len(dets)
    keys = dets["frame"].astype(np.int64) << 40 | dets["level"].astype(np.int64) << 32 | dets["wy"].astype(np.int64) << 16 | dets["wx"]
    assert (np.diff(keys) > 0).all()
    # window step: detections only on the step grid, in range
    d2, _, _ = oracle.detect_depth(casc, fr, 24, 1.25, 2, nthreads=4)
    assert len(d2) == 2 * sum(l[3] for l in oracle.plan(320, 240, 24, 1.25, 2))


def test_parse_errors():
    with pytest.raises(ValueError):
        oracle.Cascade("FDC 2\nwindow 24 24\nstages 1\nstage 1 0\nstump 1 0 0 1 1 1 0 0 0\n")
    with pytest.raises(ValueError):       # rect outside the window
        oracle.Cascade("FDC 1\nwindow 24 24\nstages 1\nstage 1 0\nstump 1 20 0 5 1 1 0 0 0\n")
    with pytest.raises(ValueError):       # weight out of range
        oracle.Cascade("FDC 1\nwindow 24 24\nstages 1\nstage 1 0\nstump 1 0 0 1 1 17 0 0 0\n")
    with pytest.raises(ValueError):       # non-finite theta
        oracle.Cascade("FDC 1\nwindow 24 24\nstages 1\nstage 1 0\nstump 1 0 0 1 1 1 nan 0 0\n")
    c = oracle.Cascade("FDC 1\nwindow 24 24\nstages 1\nstage 1 0x1.8p-1\nstump 1 0 0 1 1 1 0x1p-2 -1 1\n")
    assert c.n_stages == 1 and c.n_stumps == 1


# ---------------------------------------------------------------- c9: planted faces
@pytest.mark.parametrize("cfg,W,H,s,mfl", [(1, 320, 240, 1.25, 8), (2, 640, 480, 1.2, 12)])
def test_planted_faces_detected_iou1(cfg, W, H, s, mfl):
    casc = oracle.Cascade.from_file(os.path.join(ROOT, "cascades", f"c{cfg}.fdc"))
    lv = oracle.plan(W, H, 24, s, 1)
    fr, faces = fdgen.frames(cfg, 0, 3, W, H, lv, faces="fixed", face_param=3, max_face_level=mfl)
    dets, _ = oracle.detect(casc, fr, 24, s, 1, nthreads=4)
    for i, fl in enumerate(faces):
        for (k, wx, wy, X, Y, S) in fl:
            m = (dets["frame"] == i) & (dets["level"] == k) & (dets["wx"] == wx) & (dets["wy"] == wy)
            assert m.sum() == 1, (i, k, wx, wy)
            d = dets[m][0]
            # eq. 5 S_square (IoU) of the back-projected rect vs the planted rect = 1
            assert (d["x"], d["y"], d["w"], d["h"]) == (X, Y, S, S)


# ---------------------------------------------------------------- c10: grouping (eq. 6)
def _det(frame, x, y, w, score=0.0):
    return (frame, 0, x, y, x, y, w, w, score, 1)


def test_s_eyes_closed_form():
    # equal-size windows offset by delta: S = 2 delta / (0.4 w) = 5 delta / w
    assert oracle.s_eyes((0, 0, 100, 100), (9, 0, 100, 100)) == pytest.approx(0.45, abs=1e-12)
    assert oracle.s_eyes((0, 0, 100, 100), (10, 0, 100, 100)) == 0.5
    assert oracle.s_eyes((5, 5, 40, 40), (5, 5, 40, 40)) == 0.0
    assert oracle.s_eyes((0, 0, 100, 100), (0, 8, 100, 100)) == pytest.approx(0.4, abs=1e-12)


def test_group_hand_cases():
    D = oracle.DET_DTYPE
    # delta 9 merges, delta 10 does not (S = 0.5 exactly is not < 0.5)
    g = oracle.group(np.array([_det(0, 0, 0, 100, 1.0), _det(0, 9, 0, 100, 2.0)], D))
    assert len(g) == 1 and g[0]["aux"] == 2 and g[0]["score"] == 2.0 and g[0]["x"] == 5   # round(4.5) half up
    g = oracle.group(np.array([_det(0, 0, 0, 100), _det(0, 10, 0, 100)], D))
    assert len(g) == 2
    # identical windows merge; far windows never; frames never mix
    g = oracle.group(np.array([_det(0, 50, 50, 30), _det(0, 50, 50, 30), _det(0, 500, 50, 30),
                               _det(1, 50, 50, 30)], D))
    assert sorted(g["aux"].tolist()) == [1, 1, 2]
    # min_neighbors filters small clusters
    g = oracle.group(np.array([_det(0, 50, 50, 30), _det(0, 50, 50, 30), _det(0, 500, 50, 30)], D),
                     min_neighbors=2)
    assert len(g) == 1 and g[0]["aux"] == 2


def test_group_greedy_closest_pair_first():
    D = oracle.DET_DTYPE
    # a(0), b(4), c(8) at w=100: S(a,b)=S(b,c)=0.2 tie -> (a,b) first (lexicographic);
    # merged ab mean x=2 -> S(ab,c)=0.3 < 0.5 -> all three merge into one cluster
    g = oracle.group(np.array([_det(0, 0, 0, 100), _det(0, 4, 0, 100), _det(0, 8, 0, 100)], D))
    assert len(g) == 1 and g[0]["aux"] == 3 and g[0]["x"] == 4
    # a(0), b(9), c(18): S(a,b)=S(b,c)=0.45 -> (a,b) merge first (mean 4.5), then S(ab,c)=0.675 -> stop
    g = oracle.group(np.array([_det(0, 0, 0, 100), _det(0, 9, 0, 100), _det(0, 18, 0, 100)], D))
    assert sorted(g["aux"].tolist()) == [1, 2]


# ---------------------------------------------------------------- f3: compressed records (R13)
def test_packed16_hand_words():
    """f3: the compressed words of two hand-encoded stumps (tests/golden/packed16.txt)
    and their decoding back to the same stump."""
    g = {r[0]: [int(v) for v in r[1:]] for r in _golden("packed16.txt")}
    worked = ([(1, 1, 22, 22, -1), (1, 1, 11, 22, 2)], -0.5, 0.25, 0.75)
    diag = ([(2, 3, 8, 8, -1), (2, 3, 4, 4, 2), (6, 7, 4, 4, 2)], 1.5, -1.0, 0.125)
    for name, st in (("worked", worked), ("diagonal", diag)):
        w = oracle.pack16(*st)
        assert w == g[name], name
        assert oracle.unpack16(w, len(st[0])) == (st[0], st[1], st[2], st[3])


def test_binary16_codec_against_library():
    """f3: the oracle's binary16 decoder (written from the IEEE 754 definition) equals numpy's
    float16 for all 63488 finite encodings, and its encoder inverts it; values that are not
    binary16 are refused."""
    bits = np.arange(1 << 16, dtype=np.uint16)
    finite = ((bits >> 10) & 31) != 31
    ref = bits.view(np.float16).astype(np.float32)
    for b in bits[finite][::7]:
        v = oracle.half_value(int(b))
        assert np.float32(v).view(np.uint32) == ref[b].view(np.uint32), hex(b)
        h = oracle.half_bits(v)
        assert h == int(b) or (v == 0.0 and h in (0, 0x8000)), hex(b)
    for v, h in ((1.0, 0x3C00), (-2.0, 0xC000), (65504.0, 0x7BFF), (2.0 ** -24, 0x0001), (2.0 ** -14, 0x0400)):
        assert oracle.half_bits(v) == h
    for v in (0.1, 1.0 / 3.0, 65520.0, 2.0 ** -25, float("inf"), float(np.float32(1 + 2 ** -11))):
        assert oracle.half_bits(v) == -1, v


def test_packed_weights_and_fields():
    """f3: 6-bit two's-complement weights cover the parser's range [-16, 16]; every field range
    round-trips; a value outside binary16 makes the stump unpackable."""
    for wt in (-16, -9, -3, -2, -1, 1, 2, 3, 9, 16):
        rects = [(0, 0, 24, 24, wt), (23, 1, 1, 23, -wt)]
        w = oracle.pack16(rects, 0.0, -0.0, 1.0)
        assert oracle.unpack16(w, 2)[0] == rects
    assert oracle.pack16([(1, 1, 2, 2, 1)], 0.1, 0.5, 0.5) is None


def test_packed_cascade_round_trip_and_equivalence():
    """f3 workload c6q (c6 with binary16 theta/leaves, 'compress packed16'): the word stream is the
    concatenation of each stump's words, every stump decodes to the file's values, and the cascade
    detects exactly what the same text WITHOUT the compress line detects (the decoded records are
    the file's records)."""
    path = os.path.join(ROOT, "cascades", "c6q.fdc")
    text = open(path).read()
    casc = oracle.Cascade(text)
    words = oracle.cascade_words(casc)
    stumps = []
    for line in text.splitlines():
        t = line.split()
        if t and t[0] == "stump":
            nr = int(t[1])
            rects = [tuple(int(v) for v in t[2 + 5 * r: 7 + 5 * r]) for r in range(nr)]
            vals = [float.fromhex(v) for v in t[2 + 5 * nr: 5 + 5 * nr]]
            stumps.append((rects, *vals))
    assert len(stumps) == casc.n_stumps == 2913
    at = 0
    for st in stumps:
        w = oracle.pack16(*st)
        assert w is not None and list(words[at:at + len(w)]) == w
        assert oracle.unpack16(w, len(st[0])) == st
        at += len(w)
    assert at == len(words)
    plain = oracle.Cascade(text.replace("compress packed16\n", ""))
    assert len(oracle.cascade_words(plain)) == 0
    W, H, s = 320, 240, 1.25
    lv = oracle.plan(W, H, 24, s, 1)
    fr, _ = fdgen.frames(6, 3, 2, W, H, lv, faces="fixed", face_param=3, max_face_level=8)
    a, _ = oracle.detect(casc, fr, 24, s, 1, nthreads=4)
    b, _ = oracle.detect(plain, fr, 24, s, 1, nthreads=4)
    assert np.array_equal(a, b)
    # a cascade whose values are not binary16 cannot be compressed
    c1 = open(os.path.join(ROOT, "cascades", "c1.fdc")).read().replace("window 24 24\n", "window 24 24\ncompress packed16\n")
    with pytest.raises(ValueError):
        oracle.Cascade(c1)

