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
    ap.add_argument("--cascade", default="c3", choices=["c3", "c6", "c3s"],
                    help="c3: the paper-shaped 1446-stump cascade (c4 workload, default); c6: the "
                         "OpenCV-shaped 2913-stump cascade (SURVEY 8(f) f3 workload); c3s: c3 as a soft "
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


def stage_corner_counts(path: str):
    """Per stage: stump count and total distinct integral-image corners of its stumps (the
    shared-memory reads one window costs in that stage)."""
    sizes, corners = [], []
    for line in open(path):
        t = line.split()
        if not t or t[0].startswith("#"):
            continue
        if t[0] == "stage":
            sizes.append(int(t[1]))
            corners.append(0)
        elif t[0] == "stump":
            nr = int(t[1])
            pts = {}
            for r in range(nr):
                x, y, w, h, wt = (int(v) for v in t[2 + 5 * r: 7 + 5 * r])
                for (cx, cy, sg) in ((x, y, 1), (x + w, y, -1), (x, y + h, -1), (x + w, y + h, 1)):
                    pts[(cx, cy)] = pts.get((cx, cy), 0) + sg * wt
            corners[-1] += sum(1 for v in pts.values() if v != 0)
    return sizes, corners


def ops_model(counts, sizes, corners):
    """Algorithmic ops of the two K2 kernels: a window entering stage s
    costs corners[s] multiply-adds (one per distinct integral-image corner of each stump) +
    STUMP_OPS per stump + 1 stage compare; stage 1 adds the variance normalisation.  Loads and
    index arithmetic are not counted, so this is a lower bound on issued lane-instructions."""
    per = [k + STUMP_OPS * n + 1 for n, k in zip(sizes, corners)]
    ops1 = counts[0] * (VAR_OPS + per[0])
    opsd = sum(c * q for c, q in zip(counts[1:], per[1:]))
    return float(ops1), float(opsd)


def level_bytes(plan):
    """K1 algorithmic HBM bytes per frame: frame read + one write of ii and sqii (u32 each)."""
    W, H = CFG["W"], CFG["H"]
    b = W * H
    for (_f, w, h, _n) in plan:
        P = (w + 1 + 3) & ~3
        b += 2 * 4 * (h + 1) * P
    return b


def load_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def ncu_traffic():
    """Per-launch DRAM bytes (k_stage1, k_deep1 + k_tail, K1) from the committed ncu --set full
    capture, if any."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))
        return (d.get("k_stage1_dram_bytes_per_launch"), d.get("k_deep_dram_bytes_per_launch"),
                d.get("k1_dram_bytes_per_launch"))
    except Exception:
        return None, None, None


def make_frames(rank: int, n: int, plan):
    import fdgen
    levels = [(f, w, h) for (f, w, h, _n) in plan]
    fr, faces = fdgen.frames(CFG["cfg_id"], rank * n, n, CFG["W"], CFG["H"], levels, faces="poisson",
                             face_param=CFG["faces"], max_face_level=CFG["max_face_level"])
    return fr, faces


CASCADES = {"c3": ("c4", "25-stage 1446-stump cascade (cascades/c3.fdc)"),
            "c6": ("c6", "OpenCV-shaped 25-stage 2913-stump cascade (cascades/c6.fdc)"),
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
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    F = args.frames
    plan = fd.fd_pyramid_plan(CFG["W"], CFG["H"], CFG["min_size"], CFG["scale"], CFG["step"])
    frames_np, _faces = make_frames(rank, F, plan)
    h_frames = torch.from_numpy(frames_np).pin_memory()
    d_frames = h_frames.to(dev, non_blocking=False)
    casc_path = os.path.join(ROOT, "cascades", CFG["cascade"])
    casc = fd.Cascade.from_file(casc_path)
    sizes, corners = stage_corner_counts(casc_path)
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
        return dets.shape[0], grp.shape[0]

    def barrier():
        if world > 1:
            dist.barrier()

    for _ in range(args.warmup):
        step(False)
    torch.cuda.synchronize()
    sc.zero_()
    fd.fd_profile_reset(time_kernels=True)
    clk = ClockSampler(local)
    clk.start()
    barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    nraw = ngrp = 0
    for _ in range(args.steps):
        nraw, ngrp = step(True)
    e1.record(stream)
    torch.cuda.synchronize()
    barrier()
    clocks = clk.stop()
    ms = e0.elapsed_time(e1)
    prof = fd.fd_profile_read()
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    frames_total = F * world * args.steps
    value = frames_total / (ms / 1000.0)
    counts = [int(v) for v in sc.cpu().tolist()]        # this rank, all timed steps
    windows = counts[0]
    stumps = sum(c * n for c, n in zip(counts, sizes))

    # ---- rooflines.  K2 is two kernels: k_stage1 (dense first stage, 85% of the stumps) and the
    # deep path k_deep1 + k_tail (stages 2..N over the survivors).  Both are bound by instruction
    # issue (gathers + integer/fp32 compares; no contraction, no HBM bound): algorithmic ops per
    # window and stump are counted by ops_model(), the peak is one warp
    # instruction per SMSP per clock at the max SM clock.  The headline "roofline" is the K2
    # kernel with the larger measured time (the dominant one); K1 is HBM-bound.
    peaks = load_peaks()
    clk_max = float(peaks.get("sm_max_mhz", 1965.0))
    issue_peak = N_SM * ISSUE_LANES_PER_CLK_SM * clk_max * 1e6 / 1e9          # Gop/s
    smem_peak = N_SM * SMEM_B_PER_CLK_SM * clk_max * 1e6 / 1e9                 # GB/s
    ops1, opsd = ops_model(counts, sizes, corners)
    t1 = prof["cascade"][1]
    td = prof["deep"][1] + prof["tail"][1]
    n1 = max(prof["cascade"][0], 1)
    smem_deep = 4.0 * sum(c * k for c, k in zip(counts[1:], corners[1:]))
    roof1 = {"kernel": "k_stage1 (K2, stage 1)", "bound": "alu", "achieved": ops1 / (t1 / 1e3) / 1e9 if t1 else None,
             "peak": issue_peak, "unit": "Gop/s", "per_launch_ms": t1 / n1,
             "algorithmic_ops_per_launch": ops1 / n1,
             "peak_basis": f"148 SM x 4 SMSP x 32 lanes x {clk_max:.0f} MHz (1 warp-instruction issue/SMSP/clk)"}
    roofd = {"kernel": "k_deep1+k_tail (K2, stages 2..N)", "bound": "alu",
             "achieved": opsd / (td / 1e3) / 1e9 if td else None, "peak": issue_peak, "unit": "Gop/s",
             "per_launch_ms": td / n1, "algorithmic_ops_per_launch": opsd / n1,
             "smem_gbs": smem_deep / (td / 1e3) / 1e9 if td else None, "smem_peak_gbs": smem_peak,
             "peak_basis": roof1["peak_basis"]}
    for r in (roof1, roofd):
        r["frac"] = r["achieved"] / issue_peak if r["achieved"] else None
    tr_s1, tr_deep, tr_k1 = ncu_traffic()
    roof1["traffic"], roofd["traffic"] = tr_s1, tr_deep
    if CFG["cascade"] == "c3s.fdc":       # one kernel, k_soft, runs every stage
        roof1.update(kernel="k_soft (K2, all stages, soft cascade)", algorithmic_ops_per_launch=(ops1 + opsd) / n1,
                     achieved=(ops1 + opsd) / (t1 / 1e3) / 1e9 if t1 else None, traffic=None)
        roof1["frac"] = roof1["achieved"] / issue_peak if roof1["achieved"] else None
    dominant, other = (roofd, roof1) if td > t1 else (roof1, roofd)
    k1_ms = prof["colsum"][1] + prof["carry"][1] + prof["band"][1]
    k1_bytes = level_bytes(plan) * F * args.steps
    hbm = float(peaks.get("hbm_gbs", 6650.0))
    k1_ach = k1_bytes / (k1_ms / 1000.0) / 1e9 if k1_ms > 0 else None
    my_launches = sum(prof[k][0] for k in ("colsum", "carry", "band", "cascade", "deep", "tail", "dets", "group"))
    step_ms = ms / args.steps
    out = {
        "metric": METRIC, "value": value, "unit": "frames/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": step_ms, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u32+f32", "data": "synthetic",
        "config": workload_config(F, world),
        "windows_per_s": windows * world / (ms / 1000.0),
        "stumps_per_s": stumps * world / (ms / 1000.0),
        "detections_per_step": {"raw": nraw, "grouped": ngrp},
        "stage_entries_per_frame": [round(c / (F * args.steps), 1) for c in counts[:6]],
        "roofline": dominant,
        "roofline_k2_other": other,
        "roofline_k1": {"kernel": "k_marg+k_carry+k_corner+k_tile (K1)", "bound": "hbm", "achieved": k1_ach,
                        "peak": hbm, "unit": "GB/s", "frac": (k1_ach / hbm) if k1_ach else None,
                        "traffic": tr_k1, "peak_basis": "MEASURED_PEAKS.json hbm_gbs (burst copy)"},
        "kernel_ms_per_step": {k: v[1] / args.steps for k, v in prof.items() if v[0]},
        "gpu_launches": my_launches,
        "clocks": clocks,
    }

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
            t = torch.tensor([dt], dtype=torch.float64, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            dt = float(t.item())
        out["e2e"] = {"value": F * world * ne / dt, "unit": "frames/s",
                      "h2d_bytes_per_step": int(h_frames.numel()), "d2h_bytes_per_step": int(len(g) * 40),
                      "api": "fd_detect_group_host (pinned host frames -> grouped detections on host)"}

    # ---- CPU oracle baseline on a bounded sample (rank 0, N=1)
    if not args.no_cpu and world == 1:
        import oracle
        oc = oracle.Cascade.from_file(casc_path)
        cores = os.cpu_count() or 1
        ns = max(1, args.cpu_sample)
        t0 = time.perf_counter()
        for i in range(ns):
            d, _ = oracle.detect(oc, frames_np[i:i + 1], CFG["min_size"], CFG["scale"], CFG["step"], nthreads=cores)
            oracle.group(d)
        dt = time.perf_counter() - t0
        out["cpu_baseline"] = {"value": ns / dt, "unit": "frames/s", "cores": cores, "kind": "oracle",
                               "sample": f"first {ns} frames of the batch, detect + group, plain C oracle, "
                                         f"threads over (frame, level) jobs"}
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
