#!/usr/bin/env python3
"""Benchmark of the hot path: boosted Haar cascade over every window of every pyramid level.

Workload (BASELINE.json metric "1080p frames/s (all pyramid scales)", config c4): a synthetic
1080p video batch, 512 frames per GPU, Poisson(4) planted faces per frame, the paper-shaped
25-stage / 1446-stump cascade (cascades/c3.fdc), scale 1.1, step 1, min_size 24.
One step = one pass of every SURVEY 8(a) row over the batch: K1 pyramid+integral, K2 cascade
(all scales, one launch per frame group), K3 sort/back-projection, K4 grouping, and for N>1 the
NCCL gather of the detection lists.  Inputs are resident in HBM; 1.06 GB of frames per GPU is
larger than the 126 MB L2, so no flush is needed between steps.

python bench.py [--gpus N --steps K --warmup W] [--impl reference]
Under torchrun (N>1) each rank processes its own 512 global frames (weak scaling); the time is
the max over ranks of the CUDA-event time of the K steps.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

CFG = dict(W=1920, H=1080, scale=1.1, step=1, min_size=24, cascade="c3.fdc", cfg_id=4, faces=4.0,
           max_face_level=30)
METRIC = "1080p frames/s (all pyramid scales)"
SMEM_B_PER_CLK_SM = 128          # shared-memory crossbar, B300_MICROARCH.md "LDS/STS"
ISSUE_LANES_PER_CLK_SM = 128     # 4 SMSPs x 1 warp-instruction (32 lanes) issued per clock
N_SM = 148
VAR_OPS = 11                     # per window: 6 corner adds (S, Q), 576q, S*S, subtract, int->float, sqrt
STUMP_OPS = 5                    # per stump beyond its corner multiply-adds: i2f, fmul, fsetp, fsel, fadd
# SURVEY 8(d) instruction model (the roofline's algorithmic count): per window ~30 instructions of
# variance normalisation (8 corner loads + arithmetic); per stump 4 loads + 3 adds + 1 multiply per
# rectangle, then i2f, fmul, fsetp, fsel, fadd: 8 r + 5 (~21 for 2-rect, ~29 for 3-rect stumps)
SURVEY_VAR = 30
# f1 tile-local integral: per level pixel 1 square + 2 adds per plane (row and column prefix)
INTEGRAL_OPS_PER_PX = 5


def parse_args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--frames", type=int, default=512, help="frames per GPU")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-sample", type=int, default=2, help="frames timed on the CPU oracle")
    ap.add_argument("--cascade", default="c3", choices=["c3", "c6", "c6q", "c3s"],
                    help="c3: the paper-shaped 1446-stump cascade (c4 workload, default); c6: the "
                         "OpenCV-shaped 2913-stump cascade (SURVEY 8(f) f3 workload); c6q: c6 with compressed "
                         "records (f3, 'compress packed16'); c3s: c3 as a soft "
                         "cascade (SURVEY 8(f) f4, reading R8b, k_soft)")
    return ap.parse_args()


# ------------------------------------------------------------------ helpers
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, mx, reasons, power = [], [], set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            p = [x.strip() for x in ln.split(",")]
            if len(p) < 9:
                continue
            try:
                sm.append(float(p[1]))
                mx.append(float(p[2]))
                power.append(float(p[3]))
            except ValueError:
                continue
            for nm, v in zip(names, p[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        loaded = [s for s in sm if s > 0.5 * max(sm)] or sm
        return {"sm_mhz": statistics.median(loaded), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm), "power_w_max": max(power) if power else None}


def stage_shape(path: str):
    """Per stage: stump count, total distinct integral-image corners of its stumps (after the
    host merges shared rectangle corners) and total rectangles."""
    sizes, corners, rects = [], [], []
    for line in open(path):
        t = line.split()
        if not t or t[0].startswith("#"):
            continue
        if t[0] == "stage":
            sizes.append(int(t[1]))
            corners.append(0)
            rects.append(0)
        elif t[0] == "stump":
            nr = int(t[1])
            rects[-1] += nr
            pts = {}
            for r in range(nr):
                x, y, w, h, wt = (int(v) for v in t[2 + 5 * r: 7 + 5 * r])
                for (cx, cy, sg) in ((x, y, 1), (x + w, y, -1), (x, y + h, -1), (x + w, y + h, 1)):
                    pts[(cx, cy)] = pts.get((cx, cy), 0) + sg * wt
            corners[-1] += sum(1 for v in pts.values() if v != 0)
    return sizes, corners, rects


def ops_models(counts, sizes, corners, rects, lo: int, hi: int, with_var: bool):
    """Algorithmic lane-operations of the windows entering stages [lo, hi) (counts[s] = windows
    entering stage s): the SURVEY 8(d) instruction model (8 r + 5 per stump, 30 per window of
    variance) and a lower bound that counts no loads (one multiply-add per distinct corner, 5 per
    stump, 1 stage compare, 11 per window of variance)."""
    survey = sum(counts[s] * (8 * rects[s] + 5 * sizes[s]) for s in range(lo, min(hi, len(sizes))))
    lower = sum(counts[s] * (corners[s] + STUMP_OPS * sizes[s] + 1) for s in range(lo, min(hi, len(sizes))))
    if with_var:
        survey += counts[0] * SURVEY_VAR
        lower += counts[0] * VAR_OPS
    return float(survey), float(lower)


def level_bytes(plan, f1: bool):
    """Algorithmic HBM bytes per frame of the integral-image stage: the frame read once plus one
    write of each level image (f1: u8, pitch round_up(W_k + 1, 16)) or of each padded ii and sqii
    entry (K1: u32 each)."""
    W, H = CFG["W"], CFG["H"]
    b = W * H
    for (_f, w, h, _n) in plan:
        if f1:
            b += h * ((w + 1 + 15) & ~15)
        else:
            b += 2 * 4 * (h + 1) * ((w + 1 + 3) & ~3)
    return b


def level_pixels(plan):
    return sum(w * h for (_f, w, h, _n) in plan)


def load_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def ncu_traffic(kernel: str, frames: float = 1.0):
    """DRAM read + write bytes of `kernel` for `frames` frames, from the committed ncu --set full
    capture (profiles/ncu_traffic.json: bytes per captured launch of frames_per_launch frames)."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json"))).get(kernel, {})
        return d["dram_bytes_per_launch"] / d["frames_per_launch"] * frames
    except Exception:
        return None


def cpu_model() -> str:
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ln.startswith("Model name"):
                return ln.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def make_frames(rank: int, n: int, plan):
    import fdgen
    levels = [(f, w, h) for (f, w, h, _n) in plan]
    fr, faces = fdgen.frames(CFG["cfg_id"], rank * n, n, CFG["W"], CFG["H"], levels, faces="poisson",
                             face_param=CFG["faces"], max_face_level=CFG["max_face_level"])
    return fr, faces


CASCADES = {"c3": ("c4", "25-stage 1446-stump cascade (cascades/c3.fdc)"),
            "c6": ("c6", "OpenCV-shaped 25-stage 2913-stump cascade (cascades/c6.fdc)"),
            "c6q": ("c6q", "c6 with compressed records: two 16-bit words per rectangle, binary16 theta/leaves "
                           "(cascades/c6q.fdc, 'compress packed16')"),
            "c3s": ("c4-soft", "25-stage 1446-stump soft cascade (cascades/c3s.fdc, running-sum thresholds)")}


def workload_config(frames_per_gpu: int, world: int):
    name, desc = CASCADES[CFG["cascade"][:-4]]
    return {"workload": f"{name}: synthetic 1080p video, {frames_per_gpu} frames/GPU, Poisson(4) planted faces, "
                        f"{desc}, scale 1.1, step 1, min_size 24",
            "W": CFG["W"], "H": CFG["H"], "frames_per_gpu": frames_per_gpu, "global_frames": frames_per_gpu * world,
            "scale_factor": CFG["scale"], "step": CFG["step"], "min_size": CFG["min_size"],
            "parallelism": f"frame-sharded dp{world}" if world > 1 else "single GPU",
            "l2": "inputs (1.06 GB/GPU) larger than the 126 MB L2; no flush"}


# ------------------------------------------------------------------ reference arm (CPU oracle)
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    plan = oracle.plan(CFG["W"], CFG["H"], CFG["min_size"], CFG["scale"], CFG["step"])
    casc = oracle.Cascade.from_file(os.path.join(ROOT, "cascades", CFG["cascade"]))
    frames, _ = make_frames(0, args.warmup + args.steps, plan)
    cores = os.cpu_count() or 1
    for i in range(args.warmup):
        d, _ = oracle.detect(casc, frames[i:i + 1], CFG["min_size"], CFG["scale"], CFG["step"], nthreads=cores)
        oracle.group(d)
    t0 = time.perf_counter()
    for i in range(args.warmup, args.warmup + args.steps):
        d, _ = oracle.detect(casc, frames[i:i + 1], CFG["min_size"], CFG["scale"], CFG["step"], nthreads=cores)
        oracle.group(d)
    dt = time.perf_counter() - t0
    v = args.steps / dt
    out = {"impl": "reference", "metric": METRIC, "value": v, "unit": "frames/s", "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * dt / args.steps,
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32+f32",
           "data": "synthetic", "config": workload_config(args.frames, 1),
           "cpu_baseline": {"value": v, "unit": "frames/s", "cores": cores, "kind": "oracle",
                            "sample": f"1 frame per step ({args.steps} timed, {args.warmup} warm-up) of the c4 "
                                      "workload, plain C oracle, detect + group, threads over (frame, level)"},
           "e2e": {"value": v, "unit": "frames/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)
    return 0


# ------------------------------------------------------------------ our arm
def run_ours(args):
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_orofsmh12_b200 as fd
    from paper_conf_icpp_orofsmh12_b200 import dist as fdd

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # one process per GPU; FD_DIST_BACKEND=gloo lets ranks share a device (the 2-rank dry run of
    # this branch on a 1-GPU box, tests/test_dist.py); the detection lists then travel via the host
    backend = os.environ.get("FD_DIST_BACKEND", "nccl")
    dev_index = local % max(torch.cuda.device_count(), 1)
    torch.cuda.set_device(dev_index)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev_index))
        else:
            dist.init_process_group(backend)
    dev = torch.device("cuda", dev_index)

    def allreduce_max(x: float) -> float:
        t = torch.tensor([x], dtype=torch.float64, device=dev if backend == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())
    F = args.frames
    plan = fd.fd_pyramid_plan(CFG["W"], CFG["H"], CFG["min_size"], CFG["scale"], CFG["step"])
    frames_np, _faces = make_frames(rank, F, plan)
    h_frames = torch.from_numpy(frames_np).pin_memory()
    d_frames = h_frames.to(dev, non_blocking=False)
    casc_path = os.path.join(ROOT, "cascades", CFG["cascade"])
    casc = fd.Cascade.from_file(casc_path)
    sizes, corners, rects = stage_shape(casc_path)
    sc = torch.zeros(casc.n_stages + 1, dtype=torch.int64, device=dev)
    cap = 1 << 21
    stream = torch.cuda.current_stream()
    frame0 = rank * F

    def step(count: bool):
        dets = fd.fd_detect(casc, d_frames, CFG["min_size"], CFG["scale"], CFG["step"], capacity=cap,
                            stage_counts=sc if count else None)
        grp = fd.fd_group(dets, 0.5, 1)
        if world > 1:
            grp = fdd.gather_detections(fdd.globalize(grp, frame0))
        return dets, grp

    def barrier():
        if world > 1:
            dist.barrier()

    for _ in range(args.warmup):
        step(False)
    torch.cuda.synchronize()
    # ---- the timed region: no counters, no per-kernel events (launch counting only)
    fd.fd_profile_reset(time_kernels=False)
    clk = ClockSampler(dev_index)
    clk.start()
    barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    dets = grp = None
    for _ in range(args.steps):
        dets, grp = step(False)
    e1.record(stream)
    torch.cuda.synchronize()
    barrier()
    clocks = clk.stop()
    ms = e0.elapsed_time(e1)
    launches = fd.fd_profile_read()
    nraw, ngrp = int(dets.shape[0]), int(grp.shape[0])
    if world > 1:
        ms = allreduce_max(ms)
    frames_total = F * world * args.steps
    value = frames_total / (ms / 1000.0)

    # ---- untimed pass 1: per-stage counters (windows entering each stage, one step)
    sc.zero_()
    dets_c, _ = step(True)
    torch.cuda.synchronize()
    counts = [int(v) for v in sc.cpu().tolist()]        # this rank, one step
    windows = counts[0]
    stumps = sum(c * n for c, n in zip(counts, sizes))
    # ---- untimed pass 2: per-kernel device times, one step on ONE pipeline slot (FD_PIPE=0), so
    # a kernel's CUDA-event time is its own and not its overlap with the other slot
    os.environ["FD_PIPE"] = "0"
    fd.fd_profile_reset(time_kernels=True)
    step(False)
    torch.cuda.synchronize()
    prof = fd.fd_profile_read()
    del os.environ["FD_PIPE"]
    fd.fd_profile_reset(time_kernels=False)

    # ---- rooflines.  The cascade kernels are bound by instruction issue (gathers + integer /
    # fp32 compares: no contraction, so no tensor cores; per window far fewer bytes than
    # operations once a tile is on chip).  Algorithmic work = the SURVEY 8(d) instruction model
    # over the stage entries the kernel evaluates (ops_models); peak = one warp instruction per
    # SMSP per clock at the max SM clock.  The integral stage is reported against HBM.
    peaks = load_peaks()
    clk_max = float(peaks.get("sm_max_mhz", 1965.0))
    issue_peak = N_SM * ISSUE_LANES_PER_CLK_SM * clk_max * 1e6 / 1e9          # G lane-ops/s
    basis = f"148 SM x 4 SMSP x 32 lanes x {clk_max:.0f} MHz (1 warp-instruction issue/SMSP/clk)"
    ns = len(sizes)
    f1 = prof["level"][0] > 0
    soft = CFG["cascade"] == "c3s.fdc"

    def roof(kernel, t_ms, n_launch, lo, hi, with_var, extra_ops=0.0, traffic_key=None):
        sv, lb = ops_models(counts, sizes, corners, rects, lo, hi, with_var)
        sv += extra_ops
        lb += extra_ops
        r = {"kernel": kernel, "bound": "alu", "unit": "Gop/s", "peak": issue_peak, "peak_basis": basis,
             "per_launch_ms": t_ms / max(n_launch, 1), "launches_per_step": n_launch,
             "algorithmic_ops_per_launch": sv / max(n_launch, 1),
             "achieved": sv / (t_ms / 1e3) / 1e9 if t_ms else None,
             "lower_bound_ops_per_launch": lb / max(n_launch, 1),
             "achieved_lower_bound": lb / (t_ms / 1e3) / 1e9 if t_ms else None,
             "timing": "CUDA events on the launching stream, untimed one-slot pass (FD_PIPE=0)",
             "ops_model": "SURVEY 8(d): 30 per window (variance) + (8 r + 5) per stump evaluated"
                          + (f" + {INTEGRAL_OPS_PER_PX} per level pixel (tile-local integral)" if extra_ops else ""),
             "traffic": ncu_traffic(traffic_key, F / max(n_launch, 1)) if traffic_key else None}
        r["frac"] = r["achieved"] / issue_peak if r["achieved"] else None
        r["frac_lower_bound"] = r["achieved_lower_bound"] / issue_peak if r["achieved_lower_bound"] else None
        return r

    t_casc, n_casc = prof["cascade"][1], prof["cascade"][0]
    t_tail, t_deep = prof["tail"][1], prof["deep"][1]
    if f1:
        # k_f1 evaluates every stage (the few windows handed to k_tail continue there): the
        # roofline covers k_f1 + k_tail together over all stages, plus the tile-local integral
        roof_main = roof("k_f1+k_tail (K2: tile-local integral + every stage)", t_casc + t_tail, n_casc, 0, ns, True,
                         extra_ops=INTEGRAL_OPS_PER_PX * level_pixels(plan) * F, traffic_key="k_f1")
        roof_other = None
    elif soft:
        roof_main = roof("k_soft (K2, all stages, soft cascade)", t_casc, n_casc, 0, ns, True, traffic_key="k_soft")
        roof_other = None
    else:
        s0 = int(os.environ.get("FD_S0", "2"))
        roof_main = roof(f"k_stage1 (K2, stages [0, {s0}))", t_casc, n_casc, 0, s0, True, traffic_key="k_stage1")
        dname = "k_deep1" if os.environ.get("FD_DEEPQ", "1") == "0" else "k_deepq"
        roof_other = roof(f"{dname}{'+k_tail' if t_tail else ''} (K2, stages [{s0}, N))", t_deep + t_tail, n_casc,
                          s0, ns, False, traffic_key=dname)
        if roof_other["per_launch_ms"] > roof_main["per_launch_ms"]:
            roof_main, roof_other = roof_other, roof_main
    k1_names = ("level",) if f1 else ("colsum", "carry", "band")
    k1_ms = sum(prof[k][1] for k in k1_names)
    k1_bytes = level_bytes(plan, f1) * F
    hbm = float(peaks.get("hbm_gbs", 6650.0))
    k1_ach = k1_bytes / (k1_ms / 1000.0) / 1e9 if k1_ms > 0 else None
    my_launches = sum(v[0] for k, v in launches.items() if k != "sort")
    step_ms = ms / args.steps
    out = {
        "metric": METRIC, "value": value, "unit": "frames/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": step_ms, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u32+f32", "data": "synthetic",
        "config": workload_config(F, world),
        "windows_per_s": windows * world * args.steps / (ms / 1000.0),
        "stumps_per_s": stumps * world * args.steps / (ms / 1000.0),
        "detections_per_step": {"raw": nraw, "grouped": ngrp},
        "stage_entries_per_frame": [round(c / F, 1) for c in counts[:8]],
        "roofline": roof_main,
        "roofline_k1": {"kernel": "k_level (f1 level images)" if f1 else "k_marg+k_carry+k_corner+k_tile (K1)",
                        "bound": "hbm", "achieved": k1_ach, "peak": hbm, "unit": "GB/s",
                        "frac": (k1_ach / hbm) if k1_ach else None,
                        "algorithmic_bytes_per_frame": level_bytes(plan, f1),
                        "traffic_per_frame": ncu_traffic("k_level" if f1 else "k1"),
                        "peak_basis": "MEASURED_PEAKS.json hbm_gbs (burst copy)"},
        "kernel_ms_per_step_one_slot": {k: v[1] for k, v in prof.items() if v[0]},
        "gpu_launches": my_launches,
        "gpu_launches_per_step": {k: v[0] / args.steps for k, v in launches.items() if v[0]},
        "clocks": clocks,
    }
    if roof_other:
        out["roofline_k2_other"] = roof_other
    # ---- c3 (SURVEY 8(d) timing protocol): one resident 1080p frame per fd_detect call, including
    # its count read-back; median of 10 calls after 3 warm-up calls
    one = d_frames[0:1]
    for _ in range(3):
        fd.fd_detect(casc, one, CFG["min_size"], CFG["scale"], CFG["step"], capacity=cap)
    ts = []
    for _ in range(10):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        fd.fd_detect(casc, one, CFG["min_size"], CFG["scale"], CFG["step"], capacity=cap)
        b.record(stream)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    med = statistics.median(ts)
    out["c3_single_frame"] = {"frames_per_s": 1000.0 / med, "ms_median": med,
                              "what": "fd_detect on frame 0 alone per call (1 frame, 40 levels), count read-back included"}

    # ---- end to end through the public C ABI with HOST buffers (pinned), detect + group
    if not args.no_e2e:
        ne = max(1, min(args.steps, 3))
        fd.fd_detect_group_host(casc, h_frames, CFG["min_size"], CFG["scale"], CFG["step"], capacity=cap)
        barrier()
        t0 = time.perf_counter()
        for _ in range(ne):
            g, raw = fd.fd_detect_group_host(casc, h_frames, CFG["min_size"], CFG["scale"], CFG["step"],
                                             capacity=cap)
        dt = time.perf_counter() - t0
        if world > 1:
            dt = allreduce_max(dt)
        out["e2e"] = {"value": F * world * ne / dt, "unit": "frames/s",
                      "h2d_bytes_per_step": int(h_frames.numel()), "d2h_bytes_per_step": int(len(g) * 40),
                      "api": "fd_detect_group_host (pinned host frames -> grouped detections on host)"}

    # ---- CPU oracle baseline on a bounded sample (rank 0, N=1): all host cores on the first
    # frames of the batch, and one thread on the first frame.  The same frames give the parity
    # sample of the headline configuration: oracle near-threshold windows (c11) and the number of
    # detection records that differ from the GPU's.
    if not args.no_cpu and world == 1:
        import oracle
        oc = oracle.Cascade.from_file(casc_path)
        cores = os.cpu_count() or 1
        ns_cpu = max(1, args.cpu_sample)
        t0 = time.perf_counter()
        refs, near = [], 0
        for i in range(ns_cpu):
            d, nn = oracle.detect(oc, frames_np[i:i + 1], CFG["min_size"], CFG["scale"], CFG["step"], nthreads=cores)
            oracle.group(d)
            d["frame"] = i
            refs.append(d)
            near += nn
        dt = time.perf_counter() - t0
        t0 = time.perf_counter()
        d1, _ = oracle.detect(oc, frames_np[0:1], CFG["min_size"], CFG["scale"], CFG["step"], nthreads=1)
        oracle.group(d1)
        dt1 = time.perf_counter() - t0
        out["cpu_baseline"] = {"value": ns_cpu / dt, "unit": "frames/s", "cores": cores, "kind": "oracle",
                               "cpu_model": cpu_model(), "value_1_thread": 1.0 / dt1,
                               "sample": f"first {ns_cpu} frames of the batch on {cores} threads (threads over "
                                         f"(frame, level) jobs) and frame 0 on 1 thread, detect + group, plain C oracle"}
        ref = np.concatenate(refs)
        got = fd.to_numpy(dets_c)
        got = got[got["frame"] < ns_cpu]
        a_set = {tuple(r) for r in got.tolist()}
        b_set = {tuple(r) for r in ref.tolist()}
        out["parity_sample"] = {"frames": ns_cpu, "detections_oracle": int(len(ref)),
                                "identical": bool(np.array_equal(got, ref)),
                                "decision_mismatches": len(a_set ^ b_set),
                                "near_threshold_windows": near,
                                "near_threshold_rule": "oracle flag: |sum_s - T_s| <= 1e-4 at an evaluated stage or "
                                                       "|(float)f - theta*nf| <= 1e-4*max(1,|theta*nf|) (SURVEY 8(c) c11)"}
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    args = parse_args()
    CFG["cascade"] = f"{args.cascade}.fdc"
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
