"""bench.py — GStencil/s (eq. 18) of the LoRAStencil hot path on B200.

A "step" is one call of the C-ABI `lora_stencil_run` over the whole workload: T = 100 Jacobi
time steps of Box-2D49P on a 10240^2 FP64 grid (BASELINE.json configs[2], the north-star
target) unless --workload says otherwise.  value = T * prod(N_i) * n_ranks / t (GStencil/s).

    python bench.py [--gpus N --steps K --warmup W] [--workload NAME] [--engine auto|tc|rdg_cuda|direct]
    python bench.py --impl reference ...   # the CPU oracle (oracle/) on host cores, bounded sample

N > 1 runs under torch.distributed.run, one rank per GPU: weak scaling, every rank owns a slab
of the same local shape.  Halos move by the device-initiated exchange (lora_stencil_run_dist_p2p:
the stencil kernel stores its edge rows into the neighbour's halo over NVLink and signals it;
--dist nccl selects the host-issued NCCL send/recv path lora_stencil_run_dist instead).
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

METRIC = "GStencil/s FP64 per stencil at 1/2/4/8 B200; % of HBM roofline"
UNIT = "GStencil/s"
BYTES_PER_POINT = 16.0  # algorithmic HBM bytes per point per time step: read 8 + write 8
E2E_MIN_STEPS = 40      # e2e leg: steps timed at least (pipeline fill / drain amortised)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default=None,
                    help="synth config; default box2d49p-10240 at N = 1, box2d49p-40960 (BASELINE's multi-GPU shape) at N > 1")
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="multi-GPU shapes (40960^2, 1024^3): weak = fixed local slab (SURVEY §8(e): 5120 x 40960 / "
                         "128 x 1024^2, the global shape at N = 8), strong = the global shape split N ways")
    ap.add_argument("--engine", default="auto")
    ap.add_argument("--fuse", type=int, default=0)
    ap.add_argument("--per-stencil", action="store_true", help="also time the other Table II kernels (NEXT-3)")
    ap.add_argument("--no-configs", action="store_true", help="skip the per-config records of the BASELINE configs")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-inflight", type=int, default=3,
                    help="independent problems in flight in the e2e run (one plan + stream each)")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-engines", action="store_true", help="skip the per-engine comparison on the workload")
    ap.add_argument("--dist", default="p2p", choices=["p2p", "nccl"],
                    help="halo exchange for N > 1: device-initiated (kernel stores into the neighbour's halo) or NCCL")
    ap.add_argument("--force-dist", action="store_true",
                    help="use lora_stencil_run_dist even on one rank (exercises the slab path; LORA_DIST_SPLIT=1 "
                         "additionally forces the overlapped edge/interior split)")
    return ap.parse_args()


# ------------------------------------------------------------------ clocks (NVML) during the timed region
_REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
            0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
            0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}


class ClockSampler:
    def __init__(self, index):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _loop(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in _REASONS.items():
                    if r & bit and bit != 0x1:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.02)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._loop, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.nv:
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons)}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def load_fp64_peak():
    """Measured FP64 pipe peak (lane-ops/s: one DFMA/DADD/DMUL per lane = 1) from the newest committed
    profiles/*_fp64_peak.json (tools/fp64_peak.py); else the nominal 148 SMs x 64 FP64 lanes/clk x
    1.965 GHz (B200_PROFILING.md unit counts), saying which."""
    import glob
    fs = sorted(glob.glob(os.path.join(ROOT, "profiles", "*_fp64_peak.json")))
    if fs:
        d = json.load(open(fs[-1]))
        return float(d["ops"]["dfma_uniform"]["lane_ops_per_s"]), f"measured: {os.path.relpath(fs[-1], ROOT)} (DFMA, uniform weight operand)"
    return 148 * 64 * 1.965e9, "derived: 148 SMs x 64 FP64 lanes/clk x 1.965 GHz (no measured FP64 peak committed)"


def roofline_views(info, shape, T, fuse, t_run, hbm_peak, hbm_src, fp64_peak, fp64_src, world=1):
    """Two rooflines of the dominant (stencil) kernel from one timed run of T steps:
    hbm : ALGORITHMIC bytes per launch (16/k B per point-step x k steps = 16 B per point
          per launch, one read + one write of the grid) / average launch time, vs the measured copy BW;
    fp64: ALGORITHMIC FP64 lane-ops per launch (the plan's per-point FP64 instruction count of the
          chosen rank-1 form, e.g. 25 for the Box-2D49P row-pair split, x points x k; redundant halo
          recomputation NOT counted) / average launch time, vs the measured FP64 pipe peak.
    `bound` is the view with the larger fraction (the resource the kernel runs closest to)."""
    pts = float(np.prod(shape))
    n_launch = -(-T // fuse)
    avg = t_run / n_launch
    hb = BYTES_PER_POINT * pts
    hbm = {"bound": "hbm", "achieved": hb / avg / 1e9, "peak": hbm_peak, "unit": "GB/s",
           "frac": hb / avg / 1e9 / hbm_peak, "peak_source": hbm_src, "algorithmic_bytes_per_launch": hb}
    ops = info["fma_per_point_issued"] * pts * (T / n_launch)
    fp = {"bound": "alu", "achieved": ops / avg / 1e9, "peak": fp64_peak / 1e9, "unit": "GFP64-op/s",
          "frac": ops / avg / fp64_peak, "peak_source": fp64_src,
          "fp64_ops_per_point_step": info["fma_per_point_issued"], "algorithmic_ops_per_launch": ops,
          "note": "one FP64 lane-op = one DFMA, DADD or DMUL on one lane (the pipe's issue unit)"}
    roof = dict(fp if fp["frac"] > hbm["frac"] else hbm)
    roof.update({"avg_launch_ms": avg * 1e3, "launches_per_run": n_launch, "views": {"hbm": hbm, "fp64": fp},
                 "gstencil_roofline_hbm_unfused": hbm_peak / BYTES_PER_POINT * world,
                 "gstencil_ceiling": min(hbm_peak * fuse / BYTES_PER_POINT, fp64_peak / 1e9 / info["fma_per_point_issued"]),
                 "gstencil_ceiling_note": "min(HBM at 16/k B per point-step, FP64 peak / ops per point-step)"})
    return roof


def ncu_traffic(workload, engine):
    """dram bytes per launch from the committed ncu --set full summary, if one matches."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None
    d = json.load(open(p))
    return d.get(f"{workload}/{engine}")


def cpu_oracle_sample(W, cfg, budget_s=15.0):
    """The oracle as it stands, on all host cores, on a bounded sample of the workload: a band of
    full-width rows (2D) or planes (3D) of the same grid, stepped the workload's T times; the band
    height is sized from a one-step probe so that the sample takes about budget_s."""
    import oracle
    import synth
    h = cfg["radius"]
    shape = list(cfg["shape"])
    probe = min(shape[0], 512 if cfg["ndim"] == 2 else 16)
    pshape = [probe] + shape[1:]
    g = synth.grid(tuple(n + 2 * h for n in pshape), cfg["seed"])
    t0 = time.perf_counter(); oracle.run(W, g, 3); t1 = (time.perf_counter() - t0) / 3
    T = cfg["T"]
    full = shape[0]
    rows = int(max(1, min(full, probe * budget_s / max(t1 * T, 1e-9))))
    for _ in range(2):   # the small probe overestimates the per-row cost (thread start-up): re-size once
        shape[0] = rows
        g = synth.grid(tuple(n + 2 * h for n in shape), cfg["seed"])
        t0 = time.perf_counter(); oracle.run(W, g, T); dt = time.perf_counter() - t0
        if dt >= 0.5 * budget_s or rows == full:
            break
        rows = int(max(1, min(full, rows * budget_s / max(dt, 1e-9))))
    pts = float(np.prod(shape)) * T
    return {"value": pts / dt / 1e9, "unit": UNIT, "cores": oracle.max_threads(), "kind": "oracle",
            "sample": f"{'x'.join(map(str, shape))} interior band of {cfg['name']}, {T} steps, {dt:.1f} s"}


def host_info():
    try:
        model = [l.split(":", 1)[1].strip() for l in open("/proc/cpuinfo") if l.startswith("model name")][0]
    except Exception:
        model = "?"
    return {"nproc": os.cpu_count(), "cpu_model": model}


# ------------------------------------------------------------------ reference arm: the CPU oracle
# multi-GPU shapes (BASELINE.json configs[4]) and their weak-scaling local slabs
WEAK_SLAB = {"box2d49p-40960": (5120, 40960), "box3d27p-1024": (128, 1024, 1024)}


def local_shape(name, cfg, world, rank, scaling, force_dist=False):
    """This rank's interior slab and the global interior shape.  Multi-GPU configs: weak = the fixed
    §8(e) slab per rank (global grows with N), strong = the global shape split along the slowest axis
    (uneven splits allowed).  Other configs: every rank owns the config's shape (weak)."""
    g = tuple(cfg["shape"])
    if name in WEAK_SLAB and (world > 1 or scaling == "strong" or force_dist):
        if scaling == "weak":
            loc = WEAK_SLAB[name]
            return loc, (loc[0] * world,) + tuple(loc[1:])
        n0 = g[0] // world + (1 if rank < g[0] % world else 0)
        return (n0,) + g[1:], g
    return g, (g[0] * world,) + g[1:]


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    import synth
    W, cfg = synth.config(args.workload)
    cfg["name"] = args.workload
    h = cfg["radius"]
    # size one step so that (W + K) steps take ~150 s in total
    budget = max(2.0, 150.0 / (args.steps + args.warmup))
    shape = list(cfg["shape"])
    shape[0] = min(shape[0], 128 if cfg["ndim"] == 2 else 8)
    g = synth.grid(tuple(n + 2 * h for n in shape), cfg["seed"])
    t0 = time.perf_counter(); oracle.run(W, g, 1); t1 = time.perf_counter() - t0
    Ts = int(max(1, min(cfg["T"], budget / max(t1, 1e-6))))
    for _ in range(args.warmup):
        oracle.run(W, g, Ts)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter(); oracle.run(W, g, Ts); times.append(time.perf_counter() - t0)
    tot = sum(times)
    pts = float(np.prod(shape)) * Ts
    value = pts * args.steps / tot / 1e9
    sample = f"{'x'.join(map(str, shape))} interior band of {args.workload}, {Ts} steps per bench step"
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * tot / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic (SplitMix64 grid, seeded rsym weights)",
            "impl": "reference",
            "config": {"workload": args.workload, "grid": cfg["shape"], "T": cfg["T"], "radius": h},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": oracle.max_threads(), "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "host": host_info()}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ our arm
def main():
    args = parse()
    if args.workload is None:
        args.workload = "box2d49p-40960" if int(os.environ.get("WORLD_SIZE", "1")) > 1 else "box2d49p-10240"
    if args.impl == "reference":
        return run_reference(args)
    import torch
    import torch.distributed as dist

    import paper_conf_sc_zhanglyczcy24_b200 as L
    import synth

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)

    W, cfg = synth.config(args.workload)
    cfg["name"] = args.workload
    h, T = cfg["radius"], cfg["T"]
    shape, gshape = local_shape(args.workload, cfg, world, rank, args.scaling, args.force_dist)   # this rank's slab, global grid
    padded = tuple(n + 2 * h for n in shape)
    st = L.Stencil(W, shape, engine=args.engine, fuse_k=args.fuse)
    info = st.info()
    comm = None
    ep = None          # device-initiated exchange endpoint (lora_stencil_p2p_*)
    exchange = None
    if (world > 1 or args.force_dist) and args.dist == "p2p":
        err = ""
        try:
            ep = L.lora_stencil_p2p_create(st.plan, world, rank)
            hs = [L.lora_stencil_p2p_get_handle(ep)]
            if world > 1:
                hs = [None] * world
                dist.all_gather_object(hs, L.lora_stencil_p2p_get_handle(ep))
                L.lora_stencil_p2p_connect(ep, hs[rank - 1] if rank > 0 else None,
                                           hs[rank + 1] if rank < world - 1 else None)
        except L.LoraError as e:
            err = str(e)
        ok = torch.tensor([0 if err else 1], device=dev)
        if world > 1:
            dist.all_reduce(ok, op=dist.ReduceOp.MIN)
        if int(ok.item()) == 1:
            exchange = "p2p (device-initiated: kernel stores edge rows into the neighbour's halo, per-tile step counters)"
        else:   # every rank must use the same transport
            print(f"[bench] p2p exchange unavailable on some rank ({err or 'peer'}); using NCCL", file=sys.stderr)
            if ep is not None:
                L.lora_stencil_p2p_destroy(ep)
            ep = None
            exchange = "nccl (p2p setup failed: " + (err or "on another rank") + ")"
    if (world > 1 or args.force_dist) and ep is None:
        exchange = exchange or "nccl (host-issued send/recv, boundary strips first, overlapped with the interior)"
        if world > 1:
            uid = L.lora_stencil_comm_get_id() if rank == 0 else None
            obj = [uid]
            dist.broadcast_object_list(obj, src=0)
            uid = obj[0]
        else:
            uid = b"\0" * L.lora_stencil_comm_id_size()
        comm = L.lora_stencil_comm_init(world, rank, uid)

    # seeded synthetic input (SplitMix64 over the padded array, generated on the device — bit-identical
    # to synth.grid; each rank its own seed offset); pinned host copies for the e2e leg
    x = synth.grid_torch(padded, cfg["seed"] + 1000 * rank, device=dev)
    y = torch.empty_like(x)
    host_in = x.cpu().pin_memory()
    host_out = torch.empty_like(host_in).pin_memory()
    stream = torch.cuda.current_stream(dev)
    sptr = stream.cuda_stream

    zero_copy = ep is not None
    if zero_copy:
        # zero-copy use of the exchange buffers: the slab lives in the caller-layout view of buffer 0
        # (lora_stencil_p2p_view: inside the deep-halo buffer for fused launches), the result lands in
        # view n_launch % 2 (n_launch = ceil(T / k) even: view 0 again, so each timed step continues
        # the evolution) — no copy-in / copy-out per step
        n_launch = -(-T // max(1, info["fuse_k"]))
        b0 = L.lora_stencil_p2p_view(ep, 0)

        class _Dev:
            __cuda_array_interface__ = {"shape": tuple(x.shape), "typestr": "<f8", "data": (int(b0), False),
                                        "version": 3, "strides": None}
        torch.as_tensor(_Dev(), device=dev).copy_(x)
        torch.cuda.synchronize(dev)
        bT = L.lora_stencil_p2p_view(ep, n_launch % 2)

    def step():
        if ep is not None:
            if zero_copy:
                L.lora_stencil_run_dist_p2p(st.plan, ep, b0, bT, T, sptr)
            else:
                L.lora_stencil_run_dist_p2p(st.plan, ep, x.data_ptr(), y.data_ptr(), T, sptr)
        elif comm is None:
            L.lora_stencil_run(st.plan, x.data_ptr(), y.data_ptr(), T, sptr)
        else:
            L.lora_stencil_run_dist(st.plan, comm, x.data_ptr(), y.data_ptr(), T, sptr)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        e0.record(stream)
        for _ in range(args.steps):
            step()
        e1.record(stream)
        torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    t = e0.elapsed_time(e1) / 1e3
    if world > 1:
        tt = torch.tensor([t], device=dev, dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t = float(tt.item())
    npts = torch.tensor([float(np.prod(shape))], device=dev, dtype=torch.float64)
    if world > 1:
        dist.all_reduce(npts)          # uneven strong-scaling splits: the points all ranks processed
    pts_per_step = float(npts.item()) * T
    value = pts_per_step * args.steps / t / 1e9
    # the P2P path runs the plan's fused depth (deep halos, 2D and 3D); the NCCL path too for the
    # CUDA-core engine at N > 1 (comm-owned deep-halo buffers), else it steps unfused
    fuse = info["fuse_k"] if (comm is None or (world > 1 and info["engine_name"] == "rdg_cuda")) else 1
    launches_per_step = -(-T // fuse) + 2      # stencil launches + 2 halo-copy launches
    if ep is not None:   # ceil(T/k) stencil launches + 1 halo copy + per neighbour: 2 publish, 2 wait, 1 push
        nb = (1 if rank > 0 else 0) + (1 if rank < world - 1 else 0)
        launches_per_step = -(-T // fuse) + 1 + 5 * nb

    # roofline of the dominant kernel (the stencil kernel): HBM and FP64 views (roofline_views)
    peak, peak_src = load_peaks()
    fp64_peak, fp64_src = load_fp64_peak()
    roof = roofline_views(info, shape, T, fuse, t / args.steps, peak, peak_src, fp64_peak, fp64_src, world)
    tr = ncu_traffic(args.workload, info["engine_name"])
    if tr and int(tr.get("fuse", 1)) != fuse:
        tr = None
    if tr and tr.get("fp64_lane_ops"):
        # EXECUTED FP64 lane-ops per launch (ncu op counters, incl. the redundant halo recomputation)
        ex = float(tr["fp64_lane_ops"])
        roof["views"]["fp64_executed"] = {"achieved": ex / roof["avg_launch_ms"] * 1e3 / 1e9, "peak": fp64_peak / 1e9,
                                          "unit": "GFP64-op/s",
                                          "frac": ex / (roof["avg_launch_ms"] * 1e-3) / fp64_peak,
                                          "executed_ops_per_launch": ex, "source": tr.get("fp64_lane_ops_source")}
    roof.update({"traffic": tr["bytes"] if tr else None,       # dram read+write bytes per launch (ncu --set full)
                 "traffic_source": ({k: tr[k] for k in ("kernel", "source", "fuse")} if tr else None),
                 "kernel": f"{info['engine_name']} stencil step (fuse_k={fuse})",
                 "avg_launch_note": "timed run / stencil launches per run (the 2 halo-copy launches per run, ~0.1%, included)",
                 "frac_gstencil_of_hbm_roofline": value / (peak / BYTES_PER_POINT * world)})

    # e2e: through the C-ABI with HOST buffers (H2D of the input + D2H of the result inside the region).
    # Headline = M independent problems in flight (M plans, M streams, steps round-robin): the PCIe
    # copies of some problems overlap the stencil steps of another (one problem's H2D + D2H take
    # about as long as its T steps, so M = 2 leaves no slack; M = 3 keeps the SMs fed).  "serial" =
    # one synchronous lora_stencil_run_host call per step (copies not overlapped).
    e2e = None
    if not args.no_e2e and comm is None and ep is None:
        nbytes = host_in.numel() * 8
        L.lora_stencil_run_host(st.plan, host_in.numpy(), host_out.numpy(), T, sptr)
        torch.cuda.synchronize(dev)
        t0 = time.perf_counter()
        for _ in range(args.steps):
            L.lora_stencil_run_host(st.plan, host_in.numpy(), host_out.numpy(), T, sptr)
        te_serial = time.perf_counter() - t0
        M = max(1, args.e2e_inflight)
        extra = [L.Stencil(W, shape, engine=args.engine, fuse_k=args.fuse) for _ in range(M - 1)]
        plans = [st.plan] + [e.plan for e in extra]
        streams = [torch.cuda.Stream(dev) for _ in range(M)]
        hin = [host_in] + [torch.from_numpy(synth.grid(padded, cfg["seed"] + 1000 * rank + j)).pin_memory()
                           for j in range(1, M)]
        hout = [host_out] + [torch.empty_like(host_in).pin_memory() for _ in range(1, M)]
        for j in range(M):
            L.lora_stencil_run_host_async(plans[j], hin[j], hout[j], T, streams[j].cuda_stream)
        torch.cuda.synchronize(dev)
        # the pipeline's fill (first H2D) and drain (last D2H) are a fixed ~2 x 16 ms; over K = 10 steps
        # they cost ~11 % of the window, so the e2e leg runs at least E2E_MIN_STEPS steps (steady state)
        n_e2e = max(args.steps, E2E_MIN_STEPS)
        t0 = time.perf_counter()
        for i in range(n_e2e):
            j = i % M
            L.lora_stencil_run_host_async(plans[j], hin[j], hout[j], T, streams[j].cuda_stream)
        for s_ in streams:
            s_.synchronize()
        te = time.perf_counter() - t0
        for e in extra:
            e.close()
        e2e = {"value": pts_per_step * n_e2e / te / 1e9, "unit": UNIT, "h2d_bytes_per_step": nbytes,
               "d2h_bytes_per_step": nbytes, "steps": n_e2e,
               "api": f"lora_stencil_run_host_async (pinned host buffers), {M} problems in flight on {M} streams",
               "serial": {"value": pts_per_step * args.steps / te_serial / 1e9,
                          "api": "lora_stencil_run_host, one synchronous call per step"},
               "clock": "host wall clock around the K steps"}
    elif not args.no_e2e:
        # multi-GPU e2e: every step copies this rank's slab in from pinned host memory, runs the
        # distributed sweep (the exchange path of the timed region) and copies the result back; host
        # wall clock, max over ranks
        nbytes = host_in.numel() * 8
        xin, yout = x.data_ptr(), y.data_ptr()

        def dstep():
            x.copy_(host_in, non_blocking=True)
            if ep is not None:
                L.lora_stencil_run_dist_p2p(st.plan, ep, xin, yout, T, sptr)
            else:
                L.lora_stencil_run_dist(st.plan, comm, xin, yout, T, sptr)
            host_out.copy_(y, non_blocking=True)
        dstep()
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        for _ in range(args.steps):
            dstep()
        torch.cuda.synchronize(dev)
        te = torch.tensor([time.perf_counter() - t0], device=dev, dtype=torch.float64)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        e2e = {"value": pts_per_step * args.steps / float(te.item()) / 1e9, "unit": UNIT, "h2d_bytes_per_step": nbytes,
               "d2h_bytes_per_step": nbytes,
               "api": "torch copy_ from pinned host -> lora_stencil_run_dist" + ("_p2p" if ep is not None else "") +
                      " -> copy_ to pinned host, per rank, one stream",
               "clock": "host wall clock around the K steps, max over ranks"}

    # multi-GPU: the single-GPU run the efficiency is measured against (rank 0, no exchange): weak = the
    # same local slab on one GPU, strong = the whole global grid on one GPU
    scaling_check = None
    if (world > 1 or args.force_dist) and rank == 0:
        ref_shape = shape if (args.scaling == "weak" or args.workload not in WEAK_SLAB) else gshape
        s1 = L.Stencil(W, ref_shape, engine=args.engine, fuse_k=args.fuse)
        x1 = synth.grid_torch(tuple(n + 2 * h for n in ref_shape), cfg["seed"], device=dev)
        y1 = torch.empty_like(x1)
        L.lora_stencil_run(s1.plan, x1.data_ptr(), y1.data_ptr(), T, sptr)
        torch.cuda.synchronize(dev)
        b0, b1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        b0.record(stream)
        for _ in range(max(2, min(args.steps, 5))):
            L.lora_stencil_run(s1.plan, x1.data_ptr(), y1.data_ptr(), T, sptr)
        b1.record(stream)
        torch.cuda.synchronize(dev)
        t1 = b0.elapsed_time(b1) / 1e3 / max(2, min(args.steps, 5))
        v1 = float(np.prod(ref_shape)) * T / t1 / 1e9
        scaling_check = {"single_gpu_value": v1, "single_gpu_grid": list(ref_shape), "scaling": args.scaling,
                         "efficiency": value / (world * v1),
                         "note": "weak: value / (N x one GPU on the same local slab); strong: value / (N x one GPU on "
                                 "the global grid) — informational, the driver computes its own from the per-N values"}
        s1.close()
        del x1, y1
        torch.cuda.empty_cache()
    if world > 1:
        dist.barrier()

    # per-config records: every BASELINE single-GPU config (configs[0..3]), planner defaults, seeded
    # SplitMix64 inputs generated on the device (bit-identical to synth.grid), CUDA events around each
    # run on the launching stream, L2 flushed (a 256 MB write) before each run, NVML clocks sampled
    # during the timed runs; --per-stencil adds the other Table II kernels.
    per_config = None
    if rank == 0 and world == 1 and not args.no_configs:
        per_config = {}
        names = ["heat2d-256", "box2d9p-10240", "box2d49p-10240", "heat3d-512", "box3d27p-512"]
        if args.per_stencil:
            names += ["star2d13p-10240", "heat1d-10240000", "1d5p-10240000"]
        flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
        for name in names:
            Wn, cn = synth.config(name)
            s2 = L.Stencil(Wn, cn["shape"])
            i2 = s2.info()
            xa = synth.grid_torch(cn["padded"], cn["seed"], device=dev)
            ya = torch.empty_like(xa)
            reps = 20 if np.prod(cn["shape"]) < 1e7 else 5
            for _ in range(3):
                L.lora_stencil_run(s2.plan, xa.data_ptr(), ya.data_ptr(), cn["T"], sptr)
            torch.cuda.synchronize(dev)
            ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
            with ClockSampler(local) as clk2:
                for a0, a1 in ev:
                    flush.fill_(1)
                    a0.record(stream)
                    L.lora_stencil_run(s2.plan, xa.data_ptr(), ya.data_ptr(), cn["T"], sptr)
                    a1.record(stream)
                torch.cuda.synchronize(dev)
            ts = sorted(a0.elapsed_time(a1) / 1e3 for a0, a1 in ev)
            tmed = ts[len(ts) // 2]
            gs = float(np.prod(cn["shape"])) * cn["T"] / tmed / 1e9
            rf = roofline_views(i2, cn["shape"], cn["T"], i2["fuse_k"], tmed, peak, peak_src, fp64_peak, fp64_src)
            per_config[name] = {"value": gs, "unit": UNIT, "grid": list(cn["shape"]), "T": cn["T"],
                                "ms_per_run_median": tmed * 1e3, "ms_per_run_best": ts[0] * 1e3, "runs": reps,
                                "engine": i2["engine_name"], "fuse_k": i2["fuse_k"],
                                "fp64_ops_per_point_step": i2["fma_per_point_issued"],
                                "frac_gstencil_of_hbm_roofline": gs / (peak / BYTES_PER_POINT),
                                "roofline": {k: rf[k] for k in ("bound", "achieved", "peak", "unit", "frac")} |
                                            {"views": {v: {k: rf["views"][v][k] for k in ("achieved", "peak", "unit", "frac")}
                                                       for v in rf["views"]},
                                             "gstencil_ceiling": rf["gstencil_ceiling"]},
                                "clocks": clk2.summary(), "l2": "flushed before each run (256 MB write)",
                                "weights": cn["weights"]}
            s2.close()
            del xa, ya
        del flush
        torch.cuda.empty_cache()

    # the same workload on every engine (the paper's tensor-core chain, the CUDA-core RDG, direct)
    engines = None
    if rank == 0 and world == 1 and not args.no_engines:
        engines = {}
        for eng in ("tc", "rdg_cuda", "rdg_cuda_pma", "rdg_cuda_k1", "direct"):
            try:
                if eng == "rdg_cuda_pma":   # the paper's PMA pyramid on the CUDA-core engine (LORA_RDG_PMA=1)
                    os.environ["LORA_RDG_PMA"] = "1"
                try:
                    # the PMA form at the headline's fusion depth (its own planner default is unfused)
                    s3 = L.Stencil(W, shape, engine=eng[:8] if eng.startswith("rdg_cuda") else eng,
                                   fuse_k=1 if eng == "rdg_cuda_k1" else (info["fuse_k"] if eng == "rdg_cuda_pma" else 0))
                finally:
                    os.environ.pop("LORA_RDG_PMA", None)
            except L.LoraError as ex:
                engines[eng] = {"unsupported": str(ex)}
                continue
            L.lora_stencil_run(s3.plan, x.data_ptr(), y.data_ptr(), T, sptr)
            torch.cuda.synchronize(dev)
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            for _ in range(2):
                L.lora_stencil_run(s3.plan, x.data_ptr(), y.data_ptr(), T, sptr)
            a1.record(stream)
            torch.cuda.synchronize(dev)
            ts = a0.elapsed_time(a1) / 2e3
            gs = float(np.prod(shape)) * T / ts / 1e9
            i3 = s3.info()
            # issued FP64 rate against the measured FP64 pipe peak (step-0 microbenchmark, DESIGN.md §5:
            # DMMA 36.9 TF, DFMA 33.8 TF; profiles/r01_step0_fp64_pipes.jsonl)
            rf = roofline_views(i3, shape, T, i3["fuse_k"], ts, peak, peak_src, fp64_peak, fp64_src)
            engines[eng] = {"GStencil_s": gs, "frac_hbm_roofline": gs / (peak / BYTES_PER_POINT), "fuse_k": i3["fuse_k"],
                            "fp64_ops_per_point_step": i3["fma_per_point_issued"], "ms_per_step": ts * 1e3,
                            "n_terms": i3["n_terms"],
                            "roofline_fracs": {v: rf["views"][v]["frac"] for v in rf["views"]},
                            "fp64_pipe": ("DMMA (tensor): ops = issued FMA slots incl. band padding" if eng == "tc"
                                          else "DFMA/DADD/DMUL")}
            s3.close()

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_oracle_sample(W, cfg)

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": 1e3 * t / args.steps, "higher_is_better": True,
                "scaling": args.scaling if args.workload in WEAK_SLAB else "weak", "vs_baseline": None, "dtype": "f64",
                "data": "synthetic: SplitMix64 grid in [0.5,1.5) over the padded array, seeded radially symmetric weights",
                "config": {"workload": args.workload, "grid_per_rank": list(shape), "T": T, "radius": h,
                           "ndim": cfg["ndim"], "global_grid": list(gshape),
                           "engine": info["engine_name"], "fuse_k": fuse, "n_terms": info["n_terms"],
                           "parallelism": f"slab{world}" if (comm is not None or ep is not None) else "single",
                           "exchange": exchange,
                           "l2": "inputs (%.2f GB per buffer) larger than the 126 MB L2" % (8 * np.prod(padded) / 1e9)},
                "clocks": clk.summary(), "gpu_launches": launches_per_step * args.steps,
                "roofline": roof, "cpu_baseline": cpu, "e2e": e2e,
                "fp64_ops_per_point_step": {"chosen_form": info["fma_per_point_issued"],
                                            "direct_taps": info["fma_per_point_direct"],
                                            "separable_terms": info["fma_per_point_separable"]},
                "host": host_info()}
        if per_config:
            line["configs"] = per_config
        if scaling_check:
            line["scaling_check"] = scaling_check
        if engines:
            line["engines"] = engines
        print(json.dumps(line), flush=True)
    if comm is not None:
        L.lora_stencil_comm_destroy(comm)
    if ep is not None:
        L.lora_stencil_p2p_status(ep)
        L.lora_stencil_p2p_destroy(ep)
    st.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
