"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the same seeded
inputs.  Bar (north_star): pyramid levels, integral images, window
enumeration and depth maps bit-exact; stage scores within 1e-5 relative (the kernels are
bit-exact by construction, so equality is asserted and any near-threshold window -- oracle
flag -- is counted and reported); detection sets identical."""
import math
import os

import numpy as np
import pytest

import fdgen
import oracle
import softcasc

torch = pytest.importorskip("torch")
import paper_conf_icpp_orofsmh12_b200 as fd  # noqa: E402

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CFG = {1: (320, 240, 1.25, 8), 2: (640, 480, 1.2, 12), 3: (1920, 1080, 1.1, 30)}
_casc = {}


def cascades(cfg):
    if cfg not in _casc:
        text = open(os.path.join(ROOT, "cascades", f"c{cfg}.fdc")).read()
        _casc[cfg] = (fd.Cascade(text), oracle.Cascade(text))
    return _casc[cfg]


def gen(cfg, first, n, W=None, H=None, s=None, faces="fixed", param=3):
    W0, H0, s0, mfl = CFG.get(cfg, (W, H, s, 8))
    W, H, s = W or W0, H or H0, s or s0
    lv = oracle.plan(W, H, 24, s, 1)
    fr, planted = fdgen.frames(cfg, first, n, W, H, lv, faces=faces, face_param=param, max_face_level=mfl)
    return fr, planted


def assert_scores_equal(gpu, ref, near, what):
    g = gpu.view(np.uint32)
    r = ref.view(np.uint32)
    bad = np.nonzero(g != r)[0]
    if len(bad):
        rel = np.abs(gpu[bad] - ref[bad]) / np.maximum(np.abs(ref[bad]), 1e-30)
        assert (rel <= 1e-5).all(), f"{what}: {len(bad)} scores differ beyond 1e-5 rel"
    return len(bad)


def compare_depth(casc_pair, frames, s, step=1, min_size=24):
    gc, oc = casc_pair
    d_fr = torch.from_numpy(frames).cuda()
    depth, score = fd.fd_detect_depth(gc, d_fr, min_size, s, step)
    torch.cuda.synchronize()
    od, osc, onear = oracle.detect_depth(oc, frames, min_size, s, step, nthreads=os.cpu_count())
    gd = depth.cpu().numpy()
    gs = score.cpu().numpy()
    mism = np.nonzero(gd != od)[0]
    # decisions may only differ on windows the oracle flags as near-threshold (c11)
    assert np.all(onear[mism] != 0), f"{len(mism)} depth mismatches, {int((onear[mism] == 0).sum())} unflagged"
    same = gd == od
    nd = assert_scores_equal(gs[same], osc[same], onear[same], "depth-map scores")
    print(f"windows {len(od)}, near-threshold flagged {int((onear != 0).sum())}, depth mismatches {len(mism)}, "
          f"score bit-diffs {nd}")
    return gd, od


# ------------------------------------------------------------------ K1: pyramid + integral
@pytest.mark.parametrize("cfg", [1, 2, 3])
def test_pyramid_levels_bit_exact(cfg):
    W, H, s, _ = CFG[cfg]
    fr, _ = gen(cfg, 5, 2)
    lv = fd.fd_build_pyramid(torch.from_numpy(fr).cuda(), 24, s).cpu().numpy()
    for i in range(2):
        off = 0
        for (f, wk, hk, _) in oracle.plan(W, H, 24, s, 1):
            ref = oracle.resample(fr[i], f, wk, hk)
            got = lv[i, off:off + wk * hk].reshape(hk, wk)
            assert np.array_equal(got, ref), (i, f, wk, hk)
            off += wk * hk


@pytest.mark.parametrize("W,H", [(24, 24), (7, 5), (333, 97), (129, 257), (640, 480), (1920, 1080), (3840, 2160)])
def test_integral_bit_exact(W, H):
    rng = np.random.default_rng(W * 1000 + H)
    img = rng.integers(0, 256, (3, H, W), dtype=np.uint8)
    img[1] = 255                                   # maximal values
    ii, sq = fd.fd_integral(torch.from_numpy(img).cuda())
    ii = ii.cpu().numpy().view(np.uint32)
    sq = sq.cpu().numpy().view(np.uint64)
    for i in range(3):
        rii, rsq = oracle.integral(img[i])
        assert np.array_equal(ii[i, :, : W + 1], rii)
        assert np.array_equal(sq[i, :, : W + 1], rsq)


def test_integral_pitched_input():
    rng = np.random.default_rng(3)
    big = torch.from_numpy(rng.integers(0, 256, (2, 50, 100), dtype=np.uint8)).cuda()
    view = big[:, :, 3:80]                          # row stride 100, width 77
    ii, sq = fd.fd_integral(view)
    rii, rsq = oracle.integral(np.ascontiguousarray(big[1, :, 3:80].cpu().numpy()))
    assert np.array_equal(ii[1, :, :78].cpu().numpy().view(np.uint32), rii)


# ------------------------------------------------------------------ K2: depth maps (every window)
@pytest.mark.parametrize("cfg", [1, 2])
def test_depth_maps_bit_exact_small(cfg):
    W, H, s, _ = CFG[cfg]
    fr, _ = gen(cfg, 0, 3)
    compare_depth(cascades(cfg), fr, s)


def test_depth_maps_bit_exact_1080p():
    fr, _ = gen(3, 0, 1)
    compare_depth(cascades(3), fr, 1.1)


def test_depth_maps_generic_k2(monkeypatch):
    """Step 1 runs the K2 specialised per cascade by default (fd_jit.cpp); the generic kernel
    (FD_JIT=0) must agree too."""
    monkeypatch.setenv("FD_JIT", "0")
    fr, _ = gen(2, 3, 2)
    compare_depth(cascades(2), fr, 1.2)
    fr, _ = gen(3, 0, 1)
    compare_depth(cascades(3), fr, 1.1)


# K2 schedules (fd_api.cpp run_groups): every one computes the same depth maps and detections
K2_SCHEDULES = {
    "split_default": {},                                    # K1 -> k_stage1 -> k_deep1 + k_tail (< 4 frames per group)
    "split_s0_1": {"FD_S0": "1"},                           # k_stage1 stage 1 only
    "split_two_slot": {"FD_GROUP_FRAMES": "1"},             # 3 frame groups over 2 slots/streams
    "split_one_slot": {"FD_PIPE": "0", "FD_GROUP_FRAMES": "1"},
    "deepq": {"FD_DEEPQ": "1"},                             # K1 -> k_stage1 -> k_deepq (default at >= 4 frames per group)
    "deepq_one_slot": {"FD_DEEPQ": "1", "FD_PIPE": "0", "FD_GROUP_FRAMES": "1"},
    "deepq_tail_9": {"FD_DEEPQ": "1", "FD_DQ_TAIL": "9"},   # windows entering stage 9 go to k_tail
    "deepq_s0_1": {"FD_DEEPQ": "1", "FD_S0": "1"},
    "deepq_two_slot": {"FD_DEEPQ": "1", "FD_GROUP_FRAMES": "1"},
    "deepq_2_slots": {"FD_DEEPQ": "1", "FD_DQ_SLOTS": "2", "FD_DQ_WARPS": "4"},   # slot reuse / pinning pressure (JIT only)
    "deepq_tail_3": {"FD_DEEPQ": "1", "FD_DQ_TAIL": "3"},   # windows entering stage 3 go to k_tail
    "deepq_lane_only": {"FD_DEEPQ": "1", "FD_DQ_GROUP": "0"},    # no GL > 1 lane groups
    "deepq_generic": {"FD_DEEPQ": "1", "FD_JIT_DEEPQ_STUMPS": "0"},   # no generated deep stages
    "deepq_group_all": {"FD_DEEPQ": "1", "FD_DQ_GROUP": "32"},   # the group bound clamps to 16 windows
    "deep1": {"FD_DEEPQ": "0"},                             # K1 -> k_stage1 -> k_deep1 -> k_tail
    "deep1_two_slot": {"FD_DEEPQ": "0", "FD_GROUP_FRAMES": "1"},
    "deep1_no_tail": {"FD_DEEPQ": "0", "FD_TAIL": "0"},     # k_deep1 finishes every window
    "deep1_split_stump": {"FD_DEEPQ": "0", "FD_DEEP_SPLIT": "64"},   # deep stages <= 64 windows split-stump
    "deep1_2warps": {"FD_DEEPQ": "0", "FD_K2D_THREADS": "64"},       # two-warp k_deep1 blocks
    "deep1_s_tail_3": {"FD_DEEPQ": "0", "FD_S_TAIL": "3"},  # every window alive at stage 3 through k_tail
    "f1": {"FD_F1": "1"},                                   # k_level -> k_f1 -> k_deep1<F1> -> k_tail
    "f1_no_tail": {"FD_F1": "1", "FD_TAIL": "0"},
    "f1_tail_early": {"FD_F1": "1", "FD_TAIL_N": "200"},    # most deep windows through k_tail (u8 rebuild)
    "f1_small_groups": {"FD_F1": "1", "FD_GROUP_FRAMES": "1"},
    "f1_one_slot": {"FD_F1": "1", "FD_PIPE": "0", "FD_GROUP_FRAMES": "1"},
    "f1_fused": {"FD_F1": "1", "FD_F1_SPLIT": "0"},         # k_f1 runs every stage
    "f1_fused_split_stump": {"FD_F1": "1", "FD_F1_SPLIT": "0", "FD_DEEP_SPLIT": "64"},
    "f1_fused_s_tail_1": {"FD_F1": "1", "FD_F1_SPLIT": "0", "FD_S_TAIL": "1"},   # all stage-1 survivors to k_tail
    "f1_tail_global_records": {"FD_F1": "1", "FD_TAIL_SMEM_STUMPS": "0", "FD_S_TAIL": "3"},
    "queue": {"FD_K2_QUEUE": "1"},                          # k_soft's schedule on a hard cascade
}


# variables read when a cascade's specialised program is generated (once per fd.Cascade)
JIT_GEOMETRY_ENV = {"FD_DQ_SLOTS", "FD_DQ_WARPS", "FD_DQ_GROUP", "FD_JIT_DEEPQ_STUMPS", "FD_K2D_THREADS", "FD_K2D_CTAS",
                    "FD_F1_CTAS"}


@pytest.mark.parametrize("jit", ["1", "0"])
@pytest.mark.parametrize("name", sorted(K2_SCHEDULES))
def test_k2_schedules(name, jit, monkeypatch):
    for k, v in K2_SCHEDULES[name].items():
        monkeypatch.setenv(k, v)
    monkeypatch.setenv("FD_JIT", jit)
    pair = cascades(2)
    if jit == "1" and JIT_GEOMETRY_ENV & set(K2_SCHEDULES[name]):
        pair = (fd.Cascade(open(os.path.join(ROOT, "cascades", "c2.fdc")).read()), pair[1])
    fr, _ = gen(2, 5, 3)
    compare_depth(pair, fr, 1.2)
    gc, oc = pair
    got = fd.to_numpy(fd.fd_detect(gc, torch.from_numpy(fr).cuda(), 24, 1.2, 1, capacity=1 << 20))
    ref, _ = oracle.detect(oc, fr, 24, 1.2, 1, nthreads=os.cpu_count())
    assert np.array_equal(got, ref)
    fr, _ = gen(3, 40, 1)
    compare_depth(cascades(3), fr, 1.1)


def filtered(cfg):
    """The cfg cascade with the f2 filtering stage switched on ('filter binomial3')."""
    key = ("filtered", cfg)
    if key not in _casc:
        text = open(os.path.join(ROOT, "cascades", f"c{cfg}.fdc")).read()
        text = text.replace("window 24 24\n", "window 24 24\nfilter binomial3\n", 1)
        _casc[key] = (fd.Cascade(text), oracle.Cascade(text))
    return _casc[key]


@pytest.mark.parametrize("cfg,W,H,s", [(1, 320, 240, 1.25), (2, 640, 480, 1.2), (2, 131, 517, 1.17),
                                       (2, 401, 37, 1.3), (3, 1920, 1080, 1.1)])
def test_filter_stage_bit_exact(cfg, W, H, s):
    """f2: with the binomial filtering stage the depth maps (hence K1's filtered levels and
    integral images) and the detections equal the oracle's bit for bit."""
    n = 1 if cfg == 3 else 2
    fr = np.stack([fdgen.background(cfg, 700 + i, W, H) for i in range(n)]) if (W, H) != CFG[cfg][:2] \
        else gen(cfg, 9, n)[0]
    compare_depth(filtered(cfg), fr, s)
    gc, oc = filtered(cfg)
    got = fd.to_numpy(fd.fd_detect(gc, torch.from_numpy(fr).cuda(), 24, s, 1, capacity=1 << 20))
    ref, _ = oracle.detect(oc, fr, 24, s, 1, nthreads=os.cpu_count())
    assert np.array_equal(got, ref)


def test_c6_workload_1080p():
    """f3 workload: the OpenCV-shaped 2913-stump cascade on c4 frames -- depth maps bit-exact,
    detections identical, stage counters equal to the oracle's depth histogram."""
    W, H, s = 1920, 1080, 1.1
    lv = oracle.plan(W, H, 24, s, 1)
    fr, _ = fdgen.frames(4, 100, 2, W, H, lv, faces="poisson", face_param=4, max_face_level=30)
    text = open(os.path.join(ROOT, "cascades", "c6.fdc")).read()
    pair = (fd.Cascade(text), oracle.Cascade(text))
    compare_depth(pair, fr[:1], s)
    gc, oc = pair
    sc = torch.zeros(gc.n_stages + 1, dtype=torch.int64, device="cuda")
    got = fd.to_numpy(fd.fd_detect(gc, torch.from_numpy(fr).cuda(), 24, s, 1, capacity=1 << 20, stage_counts=sc))
    ref, _ = oracle.detect(oc, fr, 24, s, 1, nthreads=os.cpu_count())
    assert np.array_equal(got, ref)
    od, _, _ = oracle.detect_depth(oc, fr, 24, s, 1, nthreads=os.cpu_count())
    assert sc.cpu().tolist() == [int((od >= k).sum()) for k in range(gc.n_stages + 1)]


def _to_packed16(text):
    """Input generation (f3): a cascade text with theta/left/right rounded to binary16 and the
    'compress packed16' line (the oracle re-checks representability when it parses it)."""
    out = []
    for line in text.splitlines():
        t = line.split()
        if t and t[0] == "window":
            out += [line, "compress packed16"]
            continue
        if t and t[0] == "stump":
            b = 2 + 5 * int(t[1])
            t[b:b + 3] = [float(np.float32(np.float16(float.fromhex(v) if "x" in v else float(v)))).hex() for v in t[b:b + 3]]
            line = " ".join(t)
        out.append(line)
    return "\n".join(out) + "\n"


@pytest.mark.parametrize("jit", ["1", "0"])
def test_c6q_compressed_1080p(jit, monkeypatch):
    """f3 (R13): the compressed 2913-stump workload c6q -- the JIT program evaluates the
    deep lane-per-window stages from the compressed records in its constant bank, the generic
    kernels from the decoded corner records; both bit-exact with the oracle (which evaluates the
    decoded records): depth maps, detections and stage counters at 1080p."""
    monkeypatch.setenv("FD_JIT", jit)
    W, H, s = 1920, 1080, 1.1
    lv = oracle.plan(W, H, 24, s, 1)
    fr, _ = fdgen.frames(4, 200, 2, W, H, lv, faces="poisson", face_param=4, max_face_level=30)
    text = open(os.path.join(ROOT, "cascades", "c6q.fdc")).read()
    pair = (fd.Cascade(text), oracle.Cascade(text))
    compare_depth(pair, fr[:1], s)
    gc, oc = pair
    sc = torch.zeros(gc.n_stages + 1, dtype=torch.int64, device="cuda")
    got = fd.to_numpy(fd.fd_detect(gc, torch.from_numpy(fr).cuda(), 24, s, 1, capacity=1 << 20, stage_counts=sc))
    ref, _ = oracle.detect(oc, fr, 24, s, 1, nthreads=os.cpu_count())
    assert np.array_equal(got, ref)
    od, _, _ = oracle.detect_depth(oc, fr, 24, s, 1, nthreads=os.cpu_count())
    assert sc.cpu().tolist() == [int((od >= k).sum()) for k in range(gc.n_stages + 1)]


@pytest.mark.parametrize("cfg", [1, 2])
def test_packed16_small_configs(cfg):
    """f3 on the c1/c2 cascades rounded to binary16 (incl. 3-rect stumps and steps): depth maps
    bit-exact; a non-binary16 cascade is refused by the library as by the oracle."""
    W, H, s, _ = CFG[cfg]
    text = _to_packed16(open(os.path.join(ROOT, "cascades", f"c{cfg}.fdc")).read())
    pair = (fd.Cascade(text), oracle.Cascade(text))
    fr, _ = gen(cfg, 50, 2)
    compare_depth(pair, fr, s)
    compare_depth(pair, fr, s, step=2)
    bad = open(os.path.join(ROOT, "cascades", f"c{cfg}.fdc")).read().replace("window 24 24\n", "window 24 24\ncompress packed16\n")
    with pytest.raises(fd.FDError):
        fd.Cascade(bad)


@pytest.mark.parametrize("cfg,n,step", [(1, 3, 1), (2, 2, 2), (3, 1, 1)])
def test_depth_histogram(cfg, n, step):
    """f4: fd_depth_histogram (Fig. 7 analytics) equals the oracle's histogram of the oracle
    depth map, and of the GPU's own depth map, exactly."""
    W, H, s, _ = CFG[cfg]
    fr, _ = gen(cfg, 2, n)
    gc, oc = cascades(cfg)
    d_fr = torch.from_numpy(fr).cuda()
    depth, _ = fd.fd_detect_depth(gc, d_fr, 24, s, step)
    hist = fd.fd_depth_histogram(depth, n, W, H, gc.n_stages, 24, s, step).cpu().numpy()
    od, _, _ = oracle.detect_depth(oc, fr, 24, s, step, nthreads=os.cpu_count())
    assert np.array_equal(hist, oracle.depth_histogram(od, n, W, H, gc.n_stages, 24, s, step))
    assert np.array_equal(hist, oracle.depth_histogram(depth.cpu().numpy(), n, W, H, gc.n_stages, 24, s, step))


@pytest.mark.parametrize("step", [2, 3, 4])
def test_depth_maps_step(step):
    fr, _ = gen(2, 7, 2)
    compare_depth(cascades(2), fr, 1.2, step)


@pytest.mark.parametrize("W,H,s", [(24, 24, 1.1), (25, 90, 1.05), (401, 37, 1.3), (131, 517, 1.17)])
def test_depth_maps_ragged_sizes(W, H, s):
    fr = np.stack([fdgen.background(2, 900 + i, W, H) for i in range(2)])
    compare_depth(cascades(2), fr, s)


@pytest.mark.parametrize("min_size", [25, 30, 48, 97])
def test_min_size_bit_exact(min_size):
    """min_size > 24 (f_0 = min_size/24, so level 0 is itself resampled and
    every back-projected rect is scaled): levels, depth maps and detection lists."""
    W, H, s = 640, 480, 1.2
    fr, _ = gen(2, 41, 2)
    lv = fd.fd_build_pyramid(torch.from_numpy(fr).cuda(), min_size, s).cpu().numpy()
    pl = oracle.plan(W, H, min_size, s, 1)
    assert pl and abs(pl[0][0] - min_size / 24.0) < 1e-15
    for i in range(2):
        off = 0
        for (f, wk, hk, _) in pl:
            assert np.array_equal(lv[i, off:off + wk * hk].reshape(hk, wk), oracle.resample(fr[i], f, wk, hk))
            off += wk * hk
    compare_depth(cascades(2), fr, s, 1, min_size)
    gc, oc = cascades(2)
    got = fd.to_numpy(fd.fd_detect(gc, torch.from_numpy(fr).cuda(), min_size, s, 1, capacity=1 << 20))
    ref, _ = oracle.detect(oc, fr, min_size, s, 1, nthreads=os.cpu_count())
    assert np.array_equal(got, ref), f"{len(got)} vs {len(ref)} detections"


@pytest.mark.parametrize("cfg,W,H,s", [(2, 320, 240, 1.02), (1, 640, 480, 1.025)])
def test_many_levels_near_max(cfg, W, H, s):
    """117 / 122 pyramid levels, close to FD_MAX_LEVELS = 128 (the plan tables, tile scheduler
    and per-level offsets at their largest): depth maps and detection lists bit-exact."""
    assert 110 < len(oracle.plan(W, H, 24, s, 1)) <= 128
    fr = np.stack([fdgen.background(cfg, 950 + i, W, H) for i in range(2)])
    compare_depth(cascades(cfg), fr, s)
    gc, oc = cascades(cfg)
    got = fd.to_numpy(fd.fd_detect(gc, torch.from_numpy(fr).cuda(), 24, s, 1, capacity=1 << 22))
    ref, _ = oracle.detect(oc, fr, 24, s, 1, nthreads=os.cpu_count())
    assert np.array_equal(got, ref), f"{len(got)} vs {len(ref)} detections"


# ------------------------------------------------------------------ detections (fd_detect)
@pytest.mark.parametrize("cfg", [1, 2, 3])
def test_detections_identical(cfg):
    W, H, s, _ = CFG[cfg]
    n = 2 if cfg == 3 else 4
    fr, planted = gen(cfg, 11, n)
    gc, oc = cascades(cfg)
    sc = torch.zeros(gc.n_stages + 1, dtype=torch.int64, device="cuda")
    got = fd.to_numpy(fd.fd_detect(gc, torch.from_numpy(fr).cuda(), 24, s, 1, capacity=1 << 20,
                                   stage_counts=sc))
    ref, nnear = oracle.detect(oc, fr, 24, s, 1, nthreads=os.cpu_count())
    assert np.array_equal(got, ref), f"{len(got)} vs {len(ref)} detections"
    # planted faces are found with IoU 1 (eq. 5)
    for i, fl in enumerate(planted):
        for (k, wx, wy, X, Y, S) in fl:
            m = (got["frame"] == i) & (got["level"] == k) & (got["wx"] == wx) & (got["wy"] == wy)
            assert m.sum() == 1 and tuple(got[m][0][["x", "y", "w", "h"]]) == (X, Y, S, S)
    # stage counters agree with the oracle's depth histogram
    od, _, _ = oracle.detect_depth(oc, fr, 24, s, 1, nthreads=os.cpu_count())
    want = [int((od >= k).sum()) for k in range(gc.n_stages + 1)]
    assert sc.cpu().tolist() == want


def _bench_shape_parity(n_frames, first=0):
    """The c4 bench configuration (1080p, Poisson(4) planted faces, c3 cascade, s = 1.1, step 1)
    in ONE fd_detect call, so the library's own frame grouping and pipeline slots are exercised
    exactly as bench.py times them.  Every frame's detections and the per-stage counters are
    compared with the oracle, and fd_group over the whole batch with oracle.group."""
    W, H, s = 1920, 1080, 1.1
    lv = oracle.plan(W, H, 24, s, 1)
    fr, _ = fdgen.frames(4, first, n_frames, W, H, lv, faces="poisson", face_param=4, max_face_level=30)
    gc, oc = cascades(3)
    sc = torch.zeros(gc.n_stages + 1, dtype=torch.int64, device="cuda")
    dets = fd.fd_detect(gc, torch.from_numpy(fr).cuda(), 24, s, 1, capacity=1 << 22, stage_counts=sc)
    got = fd.to_numpy(dets)
    want_counts = np.zeros(gc.n_stages + 1, np.int64)
    near = 0
    refs = []
    for c0 in range(0, n_frames, 8):             # oracle in chunks (depth maps of 8 frames at a time)
        chunk = fr[c0:c0 + 8]
        ref, nn = oracle.detect(oc, chunk, 24, s, 1, nthreads=os.cpu_count())
        ref["frame"] += c0
        refs.append(ref)
        near += nn
        od, _, _ = oracle.detect_depth(oc, chunk, 24, s, 1, nthreads=os.cpu_count())
        want_counts += np.array([int((od >= k).sum()) for k in range(gc.n_stages + 1)])
    ref = np.concatenate(refs)
    print(f"{n_frames} frames: {len(ref)} detections, near-threshold windows {near}, "
          f"decision mismatches {int(len(got) != len(ref) or not np.array_equal(got, ref))}")
    for i in range(n_frames):
        assert np.array_equal(got[got["frame"] == i], ref[ref["frame"] == i]), f"frame {i}"
    assert np.array_equal(got, ref)
    assert sc.cpu().numpy().tolist() == want_counts.tolist()
    grp = fd.to_numpy(fd.fd_group(dets, 0.5, 1))
    assert np.array_equal(grp, oracle.group(ref, 0.5, 1))
    return fr


def test_video_batch_1080p_bench_shape(monkeypatch):
    """48 frames in 16-frame groups (three groups over both pipeline slots and streams), every
    frame, the stage counters and the grouping checked (VERDICT r1 'weak' 1)."""
    monkeypatch.setenv("FD_GROUP_FRAMES", "16")
    _bench_shape_parity(48)


def test_video_batch_1080p_default_groups_sampled():
    """The bench's launch configuration: the default grouping (128 1080p frames per group, from
    the 12 GiB workspace budget) over 384 frames = three groups alternating over both pipeline
    slots.  Every frame runs on the GPU; the oracle checks the detections of sampled frames at
    both ends of every group (whole-batch stage counters and grouping are checked above)."""
    W, H, s = 1920, 1080, 1.1
    n = 384
    lv = oracle.plan(W, H, 24, s, 1)
    fr, _ = fdgen.frames(4, 500, n, W, H, lv, faces="poisson", face_param=4, max_face_level=30)
    gc, oc = cascades(3)
    got = fd.to_numpy(fd.fd_detect(gc, torch.from_numpy(fr).cuda(), 24, s, 1, capacity=1 << 22))
    near = 0
    for i in (0, 1, 127, 128, 129, 255, 256, 383):
        ref, nn = oracle.detect(oc, fr[i:i + 1], 24, s, 1, nthreads=os.cpu_count())
        near += nn
        g = got[got["frame"] == i].copy()
        g["frame"] = 0
        assert np.array_equal(g, ref), f"frame {i}"
    print(f"{n} frames, 8 sampled: near-threshold windows {near}, 0 decision mismatches")


def test_video_batch_1080p_small_groups(monkeypatch):
    """12 frames in groups of 4 (FD_GROUP_FRAMES=4): three groups, slot 0 used twice."""
    monkeypatch.setenv("FD_GROUP_FRAMES", "4")
    _bench_shape_parity(12, first=100)


def test_4k_sampled():
    """c5-shaped: 2 frames 3840x2160 (Poisson(4) planted faces), both checked."""
    W, H, s = 3840, 2160, 1.1
    lv = oracle.plan(W, H, 24, s, 1)
    fr, _ = fdgen.frames(5, 0, 2, W, H, lv, faces="poisson", face_param=4, max_face_level=34)
    gc, oc = cascades(3)
    got = fd.to_numpy(fd.fd_detect(gc, torch.from_numpy(fr).cuda(), 24, s, 1))
    ref, nn = oracle.detect(oc, fr, 24, s, 1, nthreads=os.cpu_count())
    print(f"4K: {len(ref)} detections, near-threshold windows {nn}")
    assert np.array_equal(got, ref)


def test_detect_host_equals_device():
    fr, _ = gen(2, 21, 3)
    gc, _ = cascades(2)
    a = fd.to_numpy(fd.fd_detect(gc, torch.from_numpy(fr).cuda(), 24, 1.2, 1))
    b = fd.fd_detect_host(gc, torch.from_numpy(fr).pin_memory(), 24, 1.2, 1)
    assert np.array_equal(a, b)


def test_capacity_error_reports_required_count():
    fr, _ = gen(1, 0, 1)
    gc, oc = cascades(1)
    ref, _ = oracle.detect(oc, fr, 24, 1.25, 1)
    with pytest.raises(fd.FDCapacityError) as e:
        fd.fd_detect(gc, torch.from_numpy(fr).cuda(), 24, 1.25, 1, capacity=3)
    assert e.value.required == len(ref)


# ------------------------------------------------------------------ special cascades
def _casc_text(stages):
    out = ["FDC 1", "window 24 24", f"stages {len(stages)}"]
    for T, stumps in stages:
        out.append(f"stage {len(stumps)} {T}")
        for rects, th, l, r in stumps:
            rs = " ".join(" ".join(str(v) for v in rc) for rc in rects)
            out.append(f"stump {len(rects)} {rs} {th} {l} {r}")
    return "\n".join(out) + "\n"


def test_all_pass_and_all_reject():
    st = ([(1, 1, 10, 10, -1), (1, 1, 5, 10, 2)], 0.1, 0.5, 0.5)
    W, H, s = 211, 157, 1.25
    fr = np.stack([fdgen.background(1, 50 + i, W, H) for i in range(2)])
    tot = sum(p[3] for p in oracle.plan(W, H, 24, s, 1))
    allpass = fd.Cascade(_casc_text([("-inf", [st, st]), ("-1e30", [st])]))
    got = fd.to_numpy(fd.fd_detect(allpass, torch.from_numpy(fr).cuda(), 24, s, 1, capacity=2 * tot))
    assert len(got) == 2 * tot
    ref, _ = oracle.detect(oracle.Cascade(_casc_text([("-inf", [st, st]), ("-1e30", [st])])), fr, 24, s, 1)
    assert np.array_equal(got, ref)
    allrej = fd.Cascade(_casc_text([("inf", [st])]))
    d, sc = fd.fd_detect_depth(allrej, torch.from_numpy(fr).cuda(), 24, s, 1)
    assert (d.cpu().numpy() == 0).all() and (sc.cpu().numpy() == 0.5).all()
    assert len(fd.fd_detect(allrej, torch.from_numpy(fr).cuda(), 24, s, 1)) == 0


@pytest.mark.parametrize("env", [{"FD_DEEPQ": "1"}, {"FD_DEEPQ": "0"}, {"FD_DEEPQ": "1", "FD_JIT": "0"},
                                 {"FD_DEEPQ": "1", "FD_DQ_TAIL": "4"},
                                 {"FD_DEEPQ": "1", "FD_DQ_SLOTS": "2", "FD_DQ_WARPS": "4"}])
def test_all_pass_deep(env, monkeypatch):
    """Every window survives every stage of a 7-stage cascade: k_deepq's batches stay full through
    every deep stage (2048 windows per tile, more than a slot's shared-memory survivor list), slots
    are reused only after all of their windows are emitted or handed to k_tail.  Detections and
    depth maps equal the oracle's."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    st = ([(1, 1, 10, 10, -1), (1, 1, 5, 10, 2)], 0.1, 0.5, 0.25)
    text = _casc_text([("-1e30", [st] * (1 + i % 3)) for i in range(7)])
    W, H, s = 301, 203, 1.2
    fr = np.stack([fdgen.background(2, 80 + i, W, H) for i in range(3)])
    tot = sum(p[3] for p in oracle.plan(W, H, 24, s, 1))
    got = fd.to_numpy(fd.fd_detect(fd.Cascade(text), torch.from_numpy(fr).cuda(), 24, s, 1, capacity=3 * tot))
    ref, _ = oracle.detect(oracle.Cascade(text), fr, 24, s, 1, nthreads=os.cpu_count())
    assert len(got) == 3 * tot and np.array_equal(got, ref)
    compare_depth((fd.Cascade(text), oracle.Cascade(text)), fr, s)


def test_worked_example_single_stump():
    # golden worked example (tests/golden/worked_example.txt) placed at window (5, 3) of a 40x30 frame
    img = np.full((30, 40), 0, np.uint8)
    img[3:27, 5 + 12:5 + 24] = 255
    st = ([(1, 1, 22, 22, -1), (1, 1, 11, 22, 2)], -0.5, 0.25, 0.75)
    c = fd.Cascade(_casc_text([("-10", [st])]))
    d, sc = fd.fd_detect_depth(c, torch.from_numpy(img[None]).cuda(), 24, 1.5, 1)
    nx = 40 - 24 + 1
    assert float(sc.cpu().numpy()[3 * nx + 5]) == 0.25       # left leaf
    oc = oracle.Cascade(_casc_text([("-10", [st])]))
    od, osc, _ = oracle.detect_depth(oc, img, 24, 1.5, 1)
    assert np.array_equal(d.cpu().numpy(), od) and np.array_equal(sc.cpu().numpy(), osc)


def test_three_rect_and_one_rect_stumps():
    stumps = [([(0, 0, 24, 24, 1)], 0.001, -0.3, 0.4),
              ([(2, 2, 10, 12, -1), (2, 2, 5, 6, 2), (7, 8, 5, 6, 2)], 0.01, 0.2, -0.7),
              ([(3, 1, 18, 20, -1), (9, 1, 6, 20, 3)], -0.02, 0.5, -0.1),
              ([(1, 1, 21, 21, -1), (8, 8, 7, 7, 9)], 0.0, 0.3, 0.3)]
    text = _casc_text([("-0.5", stumps[:2]), ("0.1", stumps[2:]), ("-0.2", stumps)])
    fr = np.stack([fdgen.background(3, 70 + i, 300, 200) for i in range(2)])
    compare_depth((fd.Cascade(text), oracle.Cascade(text)), fr, 1.15)


# ------------------------------------------------------------------ f4: soft cascade (k_soft)
def test_soft_worked_example():
    """Reading R8b, hand-computed (tests/test_oracle.py test_soft_cascade_worked_example): the
    worked-example window at (5, 3) gives leaves 0.5 then 0.25; hard: depth 1, score 0.25;
    soft: running sum 0.75 >= 0.7, depth 2, score 0.75."""
    img = np.full((30, 40), 0, np.uint8)
    img[3:27, 5 + 12:5 + 24] = 255
    edge = [(1, 1, 22, 22, -1), (1, 1, 11, 22, 2)]
    body = _casc_text([("0.4", [(edge, -0.5, 0.5, -1.0)]), ("0.7", [(edge, -0.5, 0.25, -1.0)])])
    soft = body.replace("window 24 24\n", "window 24 24\nsoft\n")
    nx = 40 - 24 + 1
    fr = torch.from_numpy(img[None]).cuda()
    d, sc = fd.fd_detect_depth(fd.Cascade(body), fr, 24, 1.5, 1)
    assert int(d.cpu()[3 * nx + 5]) == 1 and float(sc.cpu()[3 * nx + 5]) == 0.25
    d, sc = fd.fd_detect_depth(fd.Cascade(soft), fr, 24, 1.5, 1)
    assert int(d.cpu()[3 * nx + 5]) == 2 and float(sc.cpu()[3 * nx + 5]) == 0.75
    od, osc, _ = oracle.detect_depth(oracle.Cascade(soft), img, 24, 1.5, 1)
    assert np.array_equal(d.cpu().numpy(), od) and np.array_equal(sc.cpu().numpy(), osc)


@pytest.mark.parametrize("cfg,name,n_st,per_stump,W,H,s,step", [
    (1, "c1.fdc", None, False, None, None, None, 1),
    (1, "c1.fdc", None, True, None, None, None, 1),       # one-stump stages: per-stump rejection trace
    (2, "c2.fdc", None, False, None, None, None, 1),
    (2, "c2.fdc", 6, True, 131, 517, 1.17, 1),            # ragged size, 180 one-stump stages
    (2, "c2.fdc", None, False, None, None, None, 2),
    (2, "c2.fdc", 10, False, 401, 37, 1.3, 3),
])
def test_soft_depth_maps_bit_exact(cfg, name, n_st, per_stump, W, H, s, step):
    text = softcasc.soft_from(name, n_st, per_stump)
    fr, _ = gen(cfg, 21, 2, W, H, s)
    s = s or CFG[cfg][2]
    gd, od = compare_depth((fd.Cascade(text), oracle.Cascade(text)), fr, s, step)
    assert np.array_equal(gd, od) and len(np.unique(od)) >= 3


@pytest.mark.parametrize("W,H,s,min_size", [(640, 480, 1.2, 48), (320, 240, 1.02, 24)])
def test_soft_min_size_and_many_levels(W, H, s, min_size):
    """Soft cascade (R8b) with a resampled level 0 (min_size 48) and with 117 levels."""
    text = softcasc.soft_from("c2.fdc", None, False)
    fr = np.stack([fdgen.background(2, 970 + i, W, H) for i in range(2)])
    gd, od = compare_depth((fd.Cascade(text), oracle.Cascade(text)), fr, s, 1, min_size)
    assert np.array_equal(gd, od) and len(np.unique(od)) >= 3


def test_soft_bench_cascade_1080p():
    """cascades/c3s.fdc (the `bench.py --cascade c3s` workload: calibrated running-sum thresholds)
    on a 1080p frame with planted faces: depth map and scores bit-exact against the oracle."""
    text = open(os.path.join(ROOT, "cascades", "c3s.fdc")).read()
    fr, _ = gen(3, 41, 1)
    gd, od = compare_depth((fd.Cascade(text), oracle.Cascade(text)), fr, CFG[3][2])
    assert np.array_equal(gd, od) and (od == 25).any()


def test_soft_detections_1080p():
    """The full 25-stage c3 cascade as a soft cascade at 1080p: detection lists (sorted, back-
    projected, with scores) identical to the oracle, and the stage counters equal to the oracle's
    depth histogram."""
    text = softcasc.soft_from("c3.fdc")
    W, H, s, _ = CFG[3]
    fr, _ = gen(3, 31, 1)
    gc, oc = fd.Cascade(text), oracle.Cascade(text)
    sc = torch.zeros(gc.n_stages + 1, dtype=torch.int64, device="cuda")
    got = fd.to_numpy(fd.fd_detect(gc, torch.from_numpy(fr).cuda(), 24, s, 1, capacity=1 << 22, stage_counts=sc))
    ref, _ = oracle.detect(oc, fr, 24, s, 1, nthreads=os.cpu_count())
    assert len(ref) > 0 and np.array_equal(got, ref), f"{len(got)} vs {len(ref)} detections"
    od, _, _ = oracle.detect_depth(oc, fr, 24, s, 1, nthreads=os.cpu_count())
    assert sc.cpu().tolist() == [int((od >= k).sum()) for k in range(gc.n_stages + 1)]


# ------------------------------------------------------------------ K4: grouping
@pytest.mark.parametrize("cfg", [2, 3])
def test_group_matches_oracle(cfg):
    W, H, s, _ = CFG[cfg]
    fr, _ = gen(cfg, 31, 2)
    gc, oc = cascades(cfg)
    dets = fd.fd_detect(gc, torch.from_numpy(fr).cuda(), 24, s, 1)
    ref_in = fd.to_numpy(dets)
    per_frame = max(np.bincount(ref_in["frame"]).max(), 1)
    if per_frame > 1500:
        pytest.skip("too many raw detections for the O(n^3) oracle grouping")
    got = fd.to_numpy(fd.fd_group(dets, 0.5, 1))
    ref = oracle.group(ref_in, 0.5, 1)
    assert np.array_equal(got, ref)
    got2 = fd.to_numpy(fd.fd_group(dets, 0.5, 3))
    assert np.array_equal(got2, oracle.group(ref_in, 0.5, 3))


def test_group_hand_cases():
    def det(frame, x, y, w, score=0.0):
        return (frame, 0, x, y, x, y, w, w, score, 1)
    rows = [det(0, 0, 0, 100, 1.0), det(0, 9, 0, 100, 2.0), det(0, 300, 0, 100), det(0, 310, 0, 100),
            det(1, 50, 50, 30), det(1, 50, 50, 30), det(1, 500, 50, 30), det(2, 0, 0, 100), det(2, 4, 0, 100),
            det(2, 8, 0, 100)]
    a = np.array(rows, oracle.DET_DTYPE)
    t = torch.from_numpy(a.view(np.int32).reshape(-1, 10).copy()).cuda()
    got = fd.to_numpy(fd.fd_group(t, 0.5, 1))
    assert np.array_equal(got, oracle.group(a, 0.5, 1))
