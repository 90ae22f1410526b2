#!/usr/bin/env python
"""bench.py -- FEVES inter-prediction hot path (ME + INT + SME) on B200.

Metric (BASELINE.json): "1080p frames/s and candidate GSAD/s (ME+INT+SME) at
1/2/4/8 B200".  One STEP = one IPPP inter-frame ("IPPP", P:323 one new
RF per frame): INT of the newest RF || integer FSBM ME of the CF over its
n_rf RFs (41 partitions) -> SME of all 41 x n_rf MVs, i.e. every row of
SURVEY §8(a), through me_stream_push of libfeves_me.so.  Workload at N=1:
BASELINE config[2] "1080p, 4 RFs, SA 64x64, ME + INT + SME, 1 B200"; at N>1
config[3] (same frame, MB-row sharded, strong scaling).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl feves|reference]

Timing: W untimed warm-up steps after the RF ring is full; K timed steps,
each bracketed by CUDA events on the context stream, L2 flushed (a 512 MiB
write) before every timed step, barrier + synchronize around the region, max
over ranks.  ``value`` = frames/s with inputs resident in HBM; ``e2e`` = the
same through the C-ABI with pinned HOST buffers (H2D of the frame and D2H of
the quarter-pel MVs + SADs inside every step).  ``--impl reference`` times
the CPU oracle (oracle/) on a bounded MB sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "1080p frames/s and candidate GSAD/s (ME+INT+SME) at 1/2/4/8 B200"
N_SM = 148
PX_PER_CLK_SM = 256          # 64 VABSDIFF4 lanes/clk/SM x 4 px (profiles/r01/int_peaks.json)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["feves", "reference"], default="feves")
    ap.add_argument("--config", default=None, help="synth.CONFIGS key (default: by --gpus)")
    ap.add_argument("--e2e-steps", type=int, default=50)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=10.0,
                    help="reference arm: seconds of oracle wall time per step (a seeded MB sample)")
    ap.add_argument("--cpu-frame", choices=["auto", "full", "sample"], default="auto",
                    help="cpu_baseline: the oracle on ONE FULL frame on all host cores, or a seeded MB sample "
                         "(auto: full when the calibrated estimate is <= --cpu-full-max seconds)")
    ap.add_argument("--cpu-full-max", type=float, default=90.0)
    ap.add_argument("--sme-kernel", type=int, default=None, help="ME_OPT_SME_KERNEL (0 global-load, 1 staged)")
    ap.add_argument("--rf-per-cta", type=int, default=None, help="ME_OPT_RF_PER_CTA (0 = all RFs in one CTA)")
    ap.add_argument("--sme-split", type=int, default=None, help="ME_OPT_SME_SPLIT (0 auto, 1 never, 2 always)")
    ap.add_argument("--graph", type=int, default=1,
                    help="ME_OPT_GRAPH: one CUDA graph per frame (default 1; 0 = multi-stream enqueue)")
    ap.add_argument("--pipeline", type=int, default=None, help="ME_OPT_PIPELINE_RF (default: library default)")
    ap.add_argument("--me-ctas", type=int, default=None, help="ME_OPT_ME_CTAS_PER_SM")
    ap.add_argument("--fused", type=int, default=None, help="ME_OPT_FUSED_SME")
    ap.add_argument("--lam", type=int, default=0, help="f4 variant: rate term lambda (G18); 0 = the paper's SAD")
    ap.add_argument("--max-pmv", type=int, default=0,
                    help="f4 variant: predicted-MV centre (G21), predictor = the synthetic motion rounded, clamp K")
    ap.add_argument("--adaptive", action="store_true", help="N>1: re-split MB rows every frame (SURVEY §8 f3)")
    ap.add_argument("--overlap", type=int, default=None,
                    help="ME_OPT_OVERLAP_SME for the e2e stream (SME(t) co-runs with ME(t+1))")
    ap.add_argument("--exchange", choices=["peer", "collective"], default="peer",
                    help="N>1: stripe+halo pull and SME stores over peer memory ordered by stream flags "
                         "(PeerStream) or NCCL broadcast + gather (ShardedStream)")
    return ap.parse_args()


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except OSError:
        return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}, "fallback"


def graph_period(n_rf):
    """ring phases of me_stream_push (ME_OPT_GRAPH captures one graph per phase):
    lcm(n_rf + 2 frame slots, n_rf SF slots, 2 output buffers)"""
    import math
    a = (n_rf + 2) * n_rf // math.gcd(n_rf + 2, n_rf)
    return a * 2 // math.gcd(a, 2)


def workload_units(cfg, n_ref=None):
    """Algorithmic work of one frame."""
    mbc, mbr = -(-cfg.width // 16), -(-cfg.height // 16)
    n_ref = cfg.n_rf if n_ref is None else n_ref
    n_mb = mbc * mbr
    me_cands = n_mb * n_ref * cfg.sa_range ** 2           # MB-candidates (each 256 px-absdiff, 41 SADs)
    sme_px = n_mb * n_ref * 16 * 7 * 256                   # 16 sub-pel candidates x 7 modes x 256 px
    # INT algorithmic bytes: 1 B read + 15 B written per position of the padded
    # MB-grid frame (16 B/px; 33.42 MB at 1080p) -- the SF margin rows/columns are not counted
    int_bytes = 16 * (16 * mbc) * (16 * mbr)
    return dict(n_mb=n_mb, me_cands=me_cands, me_px=me_cands * 256, sme_px=sme_px,
                gsad=me_cands + sme_px / 256, int_bytes=int_bytes)


class Clocks:
    """SM clock + throttle-reason sampler for the timed region (B200_PROFILING.md clocks line):
    an NVML thread polling every 2 ms (the timed region of a default run lasts only ~20-30 ms),
    nvidia-smi -lms 50 when NVML is unavailable."""

    NAMES = {"hw_slowdown": "nvmlClocksEventReasonHwSlowdown",
             "hw_thermal_slowdown": "nvmlClocksEventReasonHwThermalSlowdown",
             "sw_thermal_slowdown": "nvmlClocksEventReasonSwThermalSlowdown",
             "sw_power_cap": "nvmlClocksEventReasonSwPowerCap"}
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.p = None
        self.th = None
        self.samples, self.mx, self.reasons = [], None, set()

    def start(self):
        import threading
        try:
            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.mx = float(pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM))
            self.stop_ev = threading.Event()

            def run():
                while not self.stop_ev.is_set():
                    try:
                        self.samples.append(float(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)))
                        r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
                        for n, attr in self.NAMES.items():
                            if r & getattr(pynvml, attr):
                                self.reasons.add(n)
                    except pynvml.NVMLError:
                        pass
                    self.stop_ev.wait(0.002)
            self.th = threading.Thread(target=run, daemon=True)
            self.th.start()
            time.sleep(0.01)
            return
        except Exception:
            self.th = None
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "50"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            time.sleep(0.3)
        except OSError:
            self.p = None

    def stop(self):
        if self.th is not None:
            self.stop_ev.set()
            self.th.join()
            sm = self.samples
            busy = [x for x in sm if x > 300] or sm
            return {"sm_mhz": statistics.median(busy) if busy else None, "sm_max_mhz": self.mx,
                    "reasons": sorted(self.reasons), "samples": len(sm), "sampler": "nvml 2 ms"}
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        out, _ = self.p.communicate(timeout=10)
        sm, mx, reasons = [], None, set()
        names = list(self.NAMES)
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0]))
                mx = float(f[1])
            except ValueError:
                continue
            for n, v in zip(names, f[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        busy = [s for s in sm if s > 300] or sm
        return {"sm_mhz": statistics.median(busy) if busy else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm), "sampler": "nvidia-smi 50 ms"}


# ----------------------------------------------------------------- reference --

class OracleSampler:
    """The oracle (as it stands, never tuned) on the bench workload: one full frame or a
    bounded seeded MB sample of it, on a given number of host threads."""

    def __init__(self, cfg, threads=None):
        import numpy as np
        import oracle
        from synth import make_workload

        oracle.build()
        self.orc, self.cfg = oracle, cfg
        self.threads = threads or os.cpu_count() or 1
        self.cf, self.rfs = make_workload(cfg)
        self.n_total = workload_units(cfg)["n_mb"]
        self.order = np.random.default_rng(1234).permutation(self.n_total).astype(np.int32)
        self.layout = oracle.sf_layout(cfg.width, cfg.height, cfg.sa_range)
        self.t_cal = None

    def calibrate(self):
        t0 = time.perf_counter()              # one MB per thread
        self.run(self.threads)
        self.t_cal = time.perf_counter() - t0

    def size_for(self, budget_s):
        if self.t_cal is None:
            self.calibrate()
        n = self.threads * max(1, round(budget_s / max(self.t_cal, 1e-3)))
        return int(min(self.n_total, n))

    def run(self, n):
        """ME + SME of n MBs (all n_rf RFs) and INT of the matching share of one RF's SF rows.
        n = n_total is one whole frame (nothing extrapolated)."""
        import numpy as np
        cfg, orc = self.cfg, self.orc
        full = n >= self.n_total
        mbs = None if full else np.sort(self.order[:n])
        pad, pitch, rows = self.layout
        int_rows = rows if full else max(1, round(rows * n / self.n_total))
        t0 = time.perf_counter()
        mv, _ = orc.me(self.cf, self.rfs, cfg.sa_range, mb_list=mbs, threads=self.threads)
        t1 = time.perf_counter()
        me_only = cfg.path == "me"                      # BASELINE configs 1-2: integer ME only
        if not me_only:
            orc.sme(self.cf, self.rfs, mv, mb_list=mbs, threads=self.threads)
        t2 = time.perf_counter()
        if not me_only:
            orc.int_planes(self.rfs[0], pad, pitch, rows, row_begin=0, row_end=int_rows, threads=self.threads)
        t3 = time.perf_counter()
        t = t3 - t0
        fps = (min(n, self.n_total) / self.n_total) / t
        what = (f"one FULL frame: {self.n_total} MBs x {cfg.n_rf} RFs ME+SME and all {rows} SF rows of one INT "
                f"(the newest RF; stream mode)" if full else
                f"{n} of {self.n_total} MBs (seeded) x {cfg.n_rf} RFs ME+SME and {int_rows} of {rows} SF rows of "
                f"one INT, extrapolated linearly (FSBM work is linear in MBs, P:260)")
        if me_only:
            what = what.replace("ME+SME", "ME").split(" and ")[0] + (" (integer ME only)" if full else
                                                                        ", extrapolated linearly")
        return {"value": fps, "unit": "frames/s", "cores": self.threads, "kind": "oracle",
                "sample": f"{what}; {t:.1f} s wall on {self.threads} thread(s)",
                "seconds": {"me": t1 - t0, "sme": t2 - t1, "int": t3 - t2, "total": t},
                "extrapolated": not full,
                "candidate_gsad_per_s": workload_units(cfg)["gsad"] * fps / 1e9}


def cpu_baseline(cfg, args):
    """cpu_baseline of the bench line: the oracle on one full frame on all host cores
    (measured, not extrapolated), plus a single-thread timing on one MB row of it."""
    s = OracleSampler(cfg)
    full = args.cpu_frame == "full"
    if args.cpu_frame == "auto":
        s.calibrate()                           # one MB per thread
        full = s.t_cal * s.n_total / s.threads <= args.cpu_full_max
    cb = s.run(s.n_total if full else s.size_for(args.cpu_budget))
    one = OracleSampler(cfg, threads=1)
    mbc = -(-cfg.width // 16)
    st = one.run(min(mbc, one.size_for(10.0)))   # a seeded sample: one MB row's worth, at most ~10 s
    cb["single_thread"] = {"value": st["value"], "unit": "frames/s", "cores": 1, "sample": st["sample"],
                           "speedup_all_cores": cb["value"] / st["value"]}
    return cb


def run_reference(args, cfg):
    """--impl reference: the oracle as it stands, on all host cores, each step a bounded seeded
    MB sample of the bench workload (about --cpu-budget s, capped so the whole warm-up + timed run
    takes ~150 s).  ms_per_step is the MEASURED wall time of one such step; value is that step's
    frames/s (sample share / wall time) -- extrapolated from the sample, as its cpu_baseline says."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    s = OracleSampler(cfg)
    n = s.size_for(min(args.cpu_budget, 150.0 / (args.steps + args.warmup)))
    walls, cb = [], None
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        cb = s.run(n)
        if i >= args.warmup:
            walls.append(time.perf_counter() - t0)
    step_s = statistics.mean(walls)
    v = (n / s.n_total) / step_s
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "frames/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": step_s * 1e3, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "u8",
            "data": "synthetic (gen-tex, seeded)", "config": config_json(cfg, args),
            "step": f"one step = the oracle on a seeded sample of {n} of {s.n_total} MBs of the frame "
                    f"({100.0 * n / s.n_total:.1f}%), all {cfg.n_rf} RFs, ME+SME+INT share",
            "cpu_baseline": {"kind": cb["kind"], "cores": cb["cores"], "sample": cb["sample"], "value": v,
                             "unit": "frames/s"},
            "e2e": {"value": v, "unit": "frames/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "candidate_gsad_per_s": workload_units(cfg)["gsad"] * v / 1e9}
    print(json.dumps(line), flush=True)


def config_json(cfg, args):
    return {"workload": cfg.name, "baseline_config_index": cfg.baseline_index, "width": cfg.width,
            "height": cfg.height, "n_rf": cfg.n_rf, "sa_range": cfg.sa_range,
            "path": "integer FSBM ME only (me_estimate)" if cfg.path == "me" else "int+me+sme (IPPP stream)",
            "partitions": 41, "parallelism": f"mb-row x{args.gpus}" + (" adaptive" if args.adaptive else "") +
            (f" ({args.exchange} exchange)" if args.gpus > 1 else ""),
            "l2": "flushed (512 MiB write) before every timed step",
            "graph": "one CUDA graph per frame (ME_OPT_GRAPH)" if args.impl == "feves" and args.graph and args.gpus == 1
            else "none",
            **({"variant": {"lambda": args.lam, "max_pmv": args.max_pmv}} if (args.lam or args.max_pmv) else {})}


# --------------------------------------------------------------------- feves --

def _all_max(x):
    """max over ranks (device tensor for NCCL, host for the gloo smoke test)"""
    import torch.distributed as dist
    if dist.get_backend() == "gloo":
        h = x.cpu()
        dist.all_reduce(h, op=dist.ReduceOp.MAX)
        return h
    dist.all_reduce(x, op=dist.ReduceOp.MAX)
    return x


def run_me_only(args, cfg, me, dev, feves):
    """BASELINE configs 1-2 ("integer ME only" / "integer FSBM ME"): one step = me_estimate of frame
    t over its n_rf previous frames (device resident, L2 flushed before each step); e2e = the same
    through the C-ABI with the new frame uploaded from pinned host memory into a device ring and the
    full-pel MVs + SADs downloaded, every step."""
    import torch
    from synth import ippp_sequence
    n_frames = cfg.n_rf + 4
    host = ippp_sequence(cfg.width, cfg.height, n_frames, 1000 + cfg.baseline_index)
    frames = [torch.from_numpy(f).to(dev) for f in host]
    pinned = [torch.from_numpy(f).pin_memory() for f in host]
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream(dev)
    out = me.new_mvs()

    def step(t):
        me.estimate(frames[t % n_frames], [frames[(t - 1 - k) % n_frames] for k in range(cfg.n_rf)], out=out)

    for t in range(cfg.n_rf, cfg.n_rf + args.warmup):
        step(t)
    torch.cuda.synchronize()
    me.set_timing(False)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    clocks = Clocks(dev.index or 0)
    clocks.start()
    for k in range(args.steps):
        flush.fill_(k & 0xff)
        ev[k][0].record(stream)
        step(cfg.n_rf + args.warmup + k)
        ev[k][1].record(stream)
    torch.cuda.synchronize()
    ck = clocks.stop()
    total_ms = sum(a.elapsed_time(b) for a, b in ev)
    fps = args.steps / (total_ms / 1e3)
    me.set_timing(True)
    me_ms = []
    for k in range(max(5, min(args.steps, 20))):
        flush.fill_(k & 0xff)
        step(cfg.n_rf + k)
        me_ms.append(me.timings()[1])
    launches = me.launches * args.steps
    # e2e: device ring of n_rf + 1 frames, H2D of the new frame + D2H of the MVs / SADs inside the region
    ring = [torch.empty_like(frames[0]) for _ in range(cfg.n_rf + 1)]
    for i in range(cfg.n_rf):
        ring[i].copy_(frames[i])
    mv_h = torch.empty(me.mv_shape() + (2,), dtype=torch.int16).pin_memory()
    sad_h = torch.empty(me.mv_shape(), dtype=torch.uint16).pin_memory()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    n_e2e = args.e2e_steps
    for i in range(n_e2e):
        t = cfg.n_rf + i
        cur = ring[t % len(ring)]
        cur.copy_(pinned[t % n_frames], non_blocking=True)
        me.estimate(cur, [ring[(t - 1 - k) % len(ring)] for k in range(cfg.n_rf)], out=out)
        mv_h.copy_(out[0], non_blocking=True)
        sad_h.copy_(out[1], non_blocking=True)
    e1.record(stream)
    torch.cuda.synchronize()
    e2e = {"value": n_e2e / (e0.elapsed_time(e1) / 1e3), "unit": "frames/s",
           "h2d_bytes_per_step": pinned[0].numel(), "d2h_bytes_per_step": mv_h.numel() * 2 + sad_h.numel() * 2,
           "api": "me_estimate (C-ABI) on a device frame ring, pinned host frame in, full-pel MVs + SADs out"}
    u = workload_units(cfg)
    pk, pk_src = peaks()
    peak_px = N_SM * PX_PER_CLK_SM * pk.get("sm_max_mhz", 1965.0) * 1e6
    me_mean = statistics.mean(me_ms)
    achieved = u["me_px"] / (me_mean / 1e3)
    return {
        "metric": METRIC, "value": fps, "unit": "frames/s", "n_gpus": 1, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "u8",
        "data": "synthetic (gen-tex: 8 sinusoids in (1.25,-0.75) px/frame motion + noise, seeded)",
        "config": dict(config_json(cfg, args), graph="none"),
        "candidate_gsad_per_s": u["me_cands"] * fps / 1e9, "px_absdiff_per_s": u["me_px"] * fps,
        "kernels_ms": {"me": me_mean, "note": "CUDA events around the ME launch (library module timer)"},
        "clocks": ck, "e2e": e2e, "gpu_launches": launches,
        "roofline": {"bound": "alu", "kernel": f"me_fsbm_kernel<{cfg.sa_range}>", "work": "px-absdiffs of ME per launch",
                     "achieved": achieved / 1e12, "peak": peak_px / 1e12, "unit": "Tpx-absdiff/s",
                     "frac": achieved / peak_px, "traffic": None,
                     "peak_source": f"148 SM x 64 VABSDIFF4 lanes/clk x 4 px x sm_max_mhz ({pk_src})"},
        "cpu_baseline": None,
    }


def run_feves(args, cfg):
    import torch
    import torch.distributed as dist

    import __graft_entry__ as ge
    ge.build()
    import paper_conf_icpp_ilicmrs14_b200 as feves
    from paper_conf_icpp_ilicmrs14_b200.shard import PeerStream, ShardedStream, stripes
    from synth import ippp_sequence

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    local = local % torch.cuda.device_count()        # FEVES_DIST_BACKEND=gloo smoke test: ranks may share a GPU
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        backend = os.environ.get("FEVES_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    me = feves.MotionEstimator(cfg.width, cfg.height, cfg.sa_range, cfg.n_rf, device=dev, max_pmv=args.max_pmv)
    if args.lam:
        me.set_lambda(args.lam)
    if args.max_pmv:                                 # G21: RF r (frame t-1-r) predicted by the synthetic motion
        pm = torch.empty((me.mb_rows * me.mb_cols, cfg.n_rf, 2), dtype=torch.int16)
        for r in range(cfg.n_rf):
            pm[:, r, 0], pm[:, r, 1] = round(-1.25 * (r + 1)), round(0.75 * (r + 1))
        pmv_dev = pm.to(dev)
        me.set_pmv(pmv_dev)
    if cfg.path == "me" and world == 1 and not (args.lam or args.max_pmv):
        line = run_me_only(args, cfg, me, dev, feves)
        if not args.no_cpu_baseline:
            line["cpu_baseline"] = cpu_baseline(cfg, args)
        print(json.dumps(line), flush=True)
        return
    r0, r1 = stripes(me.mb_rows, world)[rank]
    me.set_rows(r0, r1)      # (ShardedStream may re-split later in adaptive mode)
    for opt, val in ((me.OPT_PIPELINE_RF, args.pipeline), (me.OPT_ME_CTAS_PER_SM, args.me_ctas),
                     (me.OPT_FUSED_SME, args.fused), (me.OPT_GRAPH, args.graph if world == 1 else None),
                     (me.OPT_SME_KERNEL, args.sme_kernel), (me.OPT_RF_PER_CTA, args.rf_per_cta),
                     (me.OPT_SME_SPLIT, args.sme_split)):
        if val is not None:
            me.set_option(opt, val)
    me.set_timing(False)                 # as in the timed pass: the graphs captured during the fill are its own
    stream = torch.cuda.current_stream(dev)

    n_frames = cfg.n_rf + 4
    host = ippp_sequence(cfg.width, cfg.height, n_frames, 1000 + cfg.baseline_index)
    frames = [torch.from_numpy(f).to(dev) for f in host]
    pinned = [torch.from_numpy(f).pin_memory() for f in host]
    buf = torch.empty_like(frames[0])
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    peer = world > 1 and args.exchange == "peer"
    if world == 1:
        ss = None
    elif peer:
        # the flag-ordered peer exchange needs CUDA IPC + stream memory operations between the
        # ranks' GPUs; if the platform refuses either (checked collectively at setup), fall back to
        # the NCCL broadcast / gather exchange and say so in the line
        try:
            ss = PeerStream(me, adaptive=args.adaptive)
            ok = 1
        except Exception as e:                       # noqa: BLE001 -- any setup failure -> fallback
            print(f"PeerStream unavailable on this platform ({e}); using ShardedStream", file=sys.stderr)
            ok = 0
        flag = torch.tensor([ok], dtype=torch.int32, device=dev)
        dist.all_reduce(flag, op=dist.ReduceOp.MIN)
        if not int(flag.item()):
            peer = False
            args.exchange = "collective (peer exchange unavailable)"
            ss = ShardedStream(me, adaptive=args.adaptive)
    else:
        ss = ShardedStream(me, adaptive=args.adaptive)

    def push(t):
        if ss is not None:
            return ss.push(frames[t % n_frames], buf)
        return me.stream_push(frames[t % n_frames], out=out_dev)

    out_dev = me.new_mvs()
    me.stream_reset()
    t = 0
    # fill the RF/SF ring (P:323 ramp), capture every ring phase's graph (period lcm(n_rf+2, n_rf, 2)),
    # then the W untimed warm-up steps
    n_fill = cfg.n_rf + (2 * graph_period(cfg.n_rf) if args.graph and world == 1 else 0)
    while t < n_fill + args.warmup:
        push(t)
        t += 1
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()

    def timed(n, timers):
        """n steps, each bracketed by CUDA events on the stream the push runs on, L2 flushed
        before each; timers: the library's per-module CUDA-event timers on (one host sync per
        step to read them) or off (no instrumentation inside the step)"""
        nonlocal t
        me.set_timing(timers)
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(n)]
        mods, launches = [], 0
        for k in range(n):
            flush.fill_(k & 0xff)
            ev[k][0].record(stream)
            push(t)
            ev[k][1].record(stream)
            t += 1
            if timers:
                mods.append(me.timings())        # waits for this step's module events
            launches += me.launches
        torch.cuda.synchronize()
        return [a.elapsed_time(b) for a, b in ev], mods, launches

    # value: K steps without instrumentation; kernels_ms / roofline: a second pass with the
    # per-module timers (the events cost a few us per step, so they stay out of `value`)
    clocks = Clocks(local)
    clocks.start()
    step_ms, _, launches = timed(args.steps, False)
    ck = clocks.stop()
    tot = torch.tensor([sum(step_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        tot = _all_max(tot)
        dist.barrier()
    total_ms = float(tot.item())
    fps = args.steps / (total_ms / 1e3)
    per_rank = None
    if peer:                                         # each rank's device time per push (CUDA events)
        ms = ss.stripe_ms()[-args.steps:]
        mine = {"rank": rank, "rows": list(ss.cur[rank]), "stripe_ms_mean": statistics.mean(ms)}
        per_rank = [None] * world
        dist.all_gather_object(per_rank, mine)
    mod_ms, mod, _ = timed(max(5, min(args.steps, 20)), True)
    graph_ab = None
    if world == 1:                                   # the other ME_OPT_GRAPH setting, same protocol
        me.set_option(me.OPT_GRAPH, 0 if args.graph else 1)
        for _ in range(2 * graph_period(cfg.n_rf)):  # warm-up: capture every ring phase
            push(t)
            t += 1
        alt_ms, _, _ = timed(max(5, min(args.steps, 20)), False)
        me.set_option(me.OPT_GRAPH, args.graph)
        graph_ab = {("stream_ms_per_step" if args.graph else "graph_ms_per_step"): statistics.mean(alt_ms),
                    ("graph_ms_per_step" if args.graph else "stream_ms_per_step"): total_ms / args.steps,
                    "note": "one CUDA graph per frame (ME_OPT_GRAPH: INT || ME -> SME, frame copy and fork/join "
                            "captured once per ring phase and replayed) vs the multi-stream enqueue; the faster "
                            "one is the bench default (--graph)"}

    # INT in isolation (inside the step it overlaps ME on the side stream); the
    # library's own module timers are switched off so only the outer events bracket it
    me.set_timing(False)
    sf_scratch = me.new_sf()
    iso = []
    for k in range(max(5, min(args.steps, 50))):
        flush.fill_(k & 0xff)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        me.interpolate(frames[k % n_frames], out=sf_scratch)
        b.record(stream)
        iso.append((a, b))
    torch.cuda.synchronize()
    int_iso_ms = statistics.mean(a.elapsed_time(b) for a, b in iso)
    # the same after a READ of the 512 MiB buffer: L2 is just as cold, but holds clean lines,
    # so INT does not pay for writing back the flush's dirty lines (ncu's cache-control
    # flush is of this kind); the roofline_int line uses this one, both are reported
    iso_r = []
    for k in range(max(5, min(args.steps, 50))):
        flush.max()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        me.interpolate(frames[k % n_frames], out=sf_scratch)
        b.record(stream)
        iso_r.append((a, b))
    torch.cuda.synchronize()
    int_iso_clean_ms = statistics.mean(a.elapsed_time(b) for a, b in iso_r)
    # "stateless" INT: all n_rf RFs of a frame interpolated back to back, as
    # me_encode_frame(n_int = n_rf) does without the stream's SF ring, L2 flushed before
    sfs_all = [sf_scratch] + [me.new_sf() for _ in range(cfg.n_rf - 1)]
    iso_s = []
    for k in range(max(5, min(args.steps, 20))):
        flush.max()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for r in range(cfg.n_rf):
            me.interpolate(frames[(k + r) % n_frames], out=sfs_all[r])
        b.record(stream)
        iso_s.append((a, b))
    torch.cuda.synchronize()
    int_stateless_ms = statistics.mean(a.elapsed_time(b) for a, b in iso_s)
    del sfs_all
    del sf_scratch
    me.set_timing(True)

    # ME alone (no SME), the kernel the roofline names, in the same launch configuration
    me_only = []
    mvs_scratch = me.new_mvs()
    rf_list = [frames[(t - 1 - k) % n_frames] for k in range(cfg.n_rf)]
    for k in range(max(3, min(args.steps, 20))):
        flush.fill_(k & 0xff)
        me.estimate(frames[t % n_frames], rf_list, out=mvs_scratch)
        me_only.append(me.timings()[1])
    del mvs_scratch
    # f2 mode decision on the stream's last quarter-pel outputs (device resident)
    md_ms = None
    if world == 1:
        md = []
        for k in range(10):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            me.mode_decision(out_dev[0], out_dev[1])
            b.record(stream)
            md.append((a, b))
        torch.cuda.synchronize()
        md_ms = statistics.median(a.elapsed_time(b) for a, b in md)

    u = workload_units(cfg)
    int_ms = statistics.mean(m[0] for m in mod)
    fused = all(m[2] < 0 for m in mod)
    me_ms = statistics.mean(m[1] for m in mod)              # fused: ME + SME in one kernel
    sme_ms = None if fused else statistics.mean(m[2] for m in mod)
    me_only_ms = statistics.mean(me_only)
    stripe_frac = (me.row1 - me.row0) / me.mb_rows
    pk, pk_src = peaks()
    peak_px = N_SM * PX_PER_CLK_SM * pk.get("sm_max_mhz", 1965.0) * 1e6
    dom_px = (u["me_px"] + (u["sme_px"] if fused else 0)) * stripe_frac
    achieved_px = dom_px / (me_ms / 1e3)
    me_only_px = u["me_px"] * stripe_frac / (me_only_ms / 1e3)
    traffic = None
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            tr = json.load(f).get(cfg.name, {})
            traffic = tr.get("me_fsbm_dram_bytes_per_launch")
    except OSError:
        pass

    # ---- e2e: pinned host frame in, host MVs/SADs out, every step ----
    e2e = None
    if not args.no_e2e and world > 1:
        # sharded: rank 0 uploads the pinned frame, the ranks exchange stripes (PeerStream:
        # peer memory; ShardedStream: broadcast + gather), rank 0 downloads the assembled
        # quarter-pel MVs + SADs
        me.stream_reset()
        for i in range(cfg.n_rf + 2):
            ss.push(frames[i % n_frames], buf)
        torch.cuda.synchronize()
        dist.barrier()
        qm_h = torch.empty((me.mb_rows, me.mb_cols, cfg.n_rf, 41, 2), dtype=torch.int16).pin_memory()
        qs_h = torch.empty((me.mb_rows, me.mb_cols, cfg.n_rf, 41), dtype=torch.uint16).pin_memory()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for i in range(args.e2e_steps):
            if rank == 0 and not peer:
                buf.copy_(pinned[(cfg.n_rf + 2 + i) % n_frames], non_blocking=True)
            if peer:
                r = ss.push(pinned[(cfg.n_rf + 2 + i) % n_frames] if rank == 0 else None)
            else:
                r = ss.push(buf, buf)
            if rank == 0:
                qm_h.copy_(r[0], non_blocking=True)
                qs_h.copy_(r[1], non_blocking=True)
        e1.record(stream)
        torch.cuda.synchronize()
        tt = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
        tt = _all_max(tt)
        e2e = {"value": args.e2e_steps / (float(tt.item()) / 1e3), "unit": "frames/s",
               "h2d_bytes_per_step": pinned[0].numel(),
               "d2h_bytes_per_step": qm_h.numel() * 2 + qs_h.numel() * 2,
               "api": ("PeerStream.push (rank 0 uploads the pinned frame; each rank pulls its stripe + halo "
                       "rows over peer memory on its copy-in stream, overlapping its previous frame, and its SME "
                       "stores into rank 0's buffer; stream-ordered peer flags, no collective)" if peer else
                       "ShardedStream.push (NCCL broadcast in, per-rank me_stream_push, NCCL gather out)")
                      + ", pinned buffers on rank 0"}
    if not args.no_e2e and world == 1:
        qm_h = torch.empty(me.mv_shape() + (2,), dtype=torch.int16).pin_memory()
        qs_h = torch.empty(me.mv_shape(), dtype=torch.uint16).pin_memory()
        if args.overlap is not None:
            me.set_option(me.OPT_OVERLAP_SME, args.overlap)
        me.stream_reset()
        for i in range(cfg.n_rf + 2):
            me.stream_push(pinned[i % n_frames], out=(qm_h, qs_h))
        me.sync()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for i in range(args.e2e_steps):
            me.stream_push(pinned[(cfg.n_rf + 2 + i) % n_frames], out=(qm_h, qs_h))
        me.stream_join()                     # the last frame's D2H (copy-out stream) is inside the region
        e1.record(stream)
        me.sync()
        torch.cuda.synchronize()
        e2e_ms = e0.elapsed_time(e1)
        e2e = {"value": args.e2e_steps / (e2e_ms / 1e3), "unit": "frames/s",
               "h2d_bytes_per_step": pinned[0].numel(),
               "d2h_bytes_per_step": qm_h.numel() * 2 + qs_h.numel() * 2,
               "api": "me_stream_push(cf_on_host=1, out_on_host=1), pinned buffers, C-ABI"
                      + (", ME_OPT_OVERLAP_SME" if args.overlap else "")}

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return
    cpu = None
    if not args.no_cpu_baseline and world == 1:
        cpu = cpu_baseline(cfg, args)
    line = {
        "metric": METRIC, "value": fps, "unit": "frames/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": total_ms / args.steps,
        "ms_per_step_median": statistics.median(step_ms), "higher_is_better": True,
        "step_ms": [round(x, 4) for x in step_ms] if os.environ.get("FEVES_BENCH_STEPS") else None,
        "scaling": "strong", "vs_baseline": None, "dtype": "u8",
        "data": "synthetic (gen-tex: 8 sinusoids in (1.25,-0.75) px/frame motion + noise, seeded)",
        "config": config_json(cfg, args),
        "candidate_gsad_per_s": u["gsad"] * fps / 1e9,
        "px_absdiff_per_s": (u["me_px"] + u["sme_px"]) * fps,
        "kernels_ms": {"int": int_ms, ("me_sme_fused" if fused else "me"): me_ms, "sme": sme_ms,
                       "int_isolated": int_iso_ms, "int_isolated_clean_l2": int_iso_clean_ms,
                       "int_stateless_all_rf": int_stateless_ms, "mode_decision": md_ms,
                       "me_only_isolated": me_only_ms,
                       "note": "CUDA events around each launch on its own stream" + (
                           "; fused: INT(t-1) then one ME+SME kernel" if fused else
                           "; INT runs concurrently with ME (P:86) on a side stream")},
        "clocks": ck,
        "graph_ab": graph_ab,
        "per_rank": per_rank,
        "e2e": e2e,
        "gpu_launches": launches,
        "roofline": {"bound": "alu", "kernel": "me_fsbm_kernel<64,fused>" if fused else "me_fsbm_kernel<64>",
                     "work": "px-absdiffs of ME" + (" + SME (fused kernel)" if fused else "") + " per launch",
                     "achieved": achieved_px / 1e12,
                     "peak": peak_px / 1e12, "unit": "Tpx-absdiff/s", "frac": achieved_px / peak_px,
                     "traffic": traffic,
                     "peak_source": f"148 SM x 64 VABSDIFF4 lanes/clk x 4 px x sm_max_mhz ({pk_src} "
                                    "MEASURED_PEAKS.json); issue rate measured in profiles/r01/int_peaks.json",
                     "frac_at_observed_clock": (achieved_px / (N_SM * PX_PER_CLK_SM * ck["sm_mhz"] * 1e6))
                     if ck.get("sm_mhz") else None},
        "roofline_me_only": {"bound": "alu", "kernel": "me_fsbm_kernel<64> (ME alone, isolated, L2 flushed)",
                             "achieved": me_only_px / 1e12, "peak": peak_px / 1e12, "unit": "Tpx-absdiff/s",
                             "frac": me_only_px / peak_px},
        "roofline_int": {"bound": "hbm", "kernel": "int_tile_kernel (ME_OPT_INT_KERNEL = 1, default)",
                         "traffic_unit": "16 B per position of the padded MB-grid frame (SURVEY §8(d): 1 B read "
                                         "+ 15 B written)",
                         "limiter": "issue / latency, not HBM (ncu: the planes land in L2; DESIGN.md §6)",
                         "stateless_all_rf": {"ms": int_stateless_ms, "frames_rf": cfg.n_rf,
                                              "achieved_gbs": cfg.n_rf * u["int_bytes"] * stripe_frac /
                                              (int_stateless_ms / 1e3) / 1e9},
                         "timing": "isolated, L2 flushed by a 512 MiB read (cold, clean lines); after a 512 MiB "
                                   "write flush (dirty lines to write back) see kernels_ms.int_isolated",
                         "achieved": u["int_bytes"] * stripe_frac / (int_iso_clean_ms / 1e3) / 1e9,
                         "peak": pk.get("hbm_gbs", 6650.0), "unit": "GB/s",
                         "frac": u["int_bytes"] * stripe_frac / (int_iso_clean_ms / 1e3) / 1e9 / pk.get("hbm_gbs", 6650.0)},
        "cpu_baseline": cpu,
    }
    if sme_ms:   # SME against the same ALU roofline (its binding resource is L1 latency/wavefronts)
        sme_px_s = u["sme_px"] * stripe_frac / (sme_ms / 1e3)
        line["roofline_sme"] = {"bound": "alu", "kernel": "sme_refine_kernel", "timing": "in the step",
                                "achieved": sme_px_s / 1e12, "peak": peak_px / 1e12, "unit": "Tpx-absdiff/s",
                                "frac": sme_px_s / peak_px,
                                "note": "latency / L1-data-pipe bound, not ALU (ncu: 76% of L1 data-pipe "
                                        "wavefronts, 41% issue active; DESIGN.md §6)"}
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def main():
    args = parse()
    from synth import CONFIGS
    name = args.config or ("1080p_sa64_4rf" if args.gpus == 1 else "1080p_shard")
    cfg = CONFIGS[name]
    if args.warmup < 3:
        raise SystemExit("--warmup must be >= 3")
    if args.impl == "reference":
        run_reference(args, cfg)
    else:
        run_feves(args, cfg)


if __name__ == "__main__":
    main()
