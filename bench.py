#!/usr/bin/env python
"""bench.py — libbmr hot-path benchmark (BASELINE.json metric: Map+Group+Reduce input GB/s and
% HBM roofline, vs the CPU oracle).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C5|C4|C3|C2|C1] [--impl reference]
                    [--scaling weak|strong] [--mode SIO|SO|SI|G] [--no-map-combine] [--km-full-scan]
                    [--xchg nccl|caller|fused] [--units U]

One step = one pass of the whole hot path (tile scheduling, stage-in,
user map, emit, flush, digit histogram, onesweep passes, segment boundaries, reduce + output
assembly) over one shard of synthetic input already resident in HBM.  Default workload = C5
(WordCount, Zipf V=1M, 8 GiB per GPU, weak scaling): the configuration the metric's
"1/2/4/8 B200" is quoted on that exercises every row (C2 StringMatch is Map-only).
Prints ONE JSON line on rank 0.  Timing: W warm-up steps, then K steps bracketed by barrier +
cuda.synchronize, CUDA events on the job stream, max over ranks.  Inputs (8 GiB) exceed L2
(126 MB), so no extra flush is needed.

Multi-GPU: ``--gpus N`` without a torchrun environment re-launches this script under
``torch.distributed.run`` with N ranks (one per GPU, 127.0.0.1 rendezvous); under torchrun the
world size comes from the environment (and must equal N).  The exchange is
libbmr's own: mr_group over an NCCL communicator the library creates (``--xchg nccl``, default);
``--xchg caller`` moves the partition buffers with torch.distributed (Job.shuffle); ``--xchg
fused`` (InvertedIndex) lets the Maps store straight into the owners' receive windows through
CUDA IPC.  ``--scaling strong`` fixes the total input (C5: 64 GiB, split 64/N
GiB per GPU and processed in 8 GiB batches with the per-batch combine, MR_FLAG_BATCH_COMBINE);
the default ``weak`` gives every GPU the 1-GPU configuration's shard.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOADS = {
    # name: (workload, description, pages-or-points per GPU)
    "C1": ("wc", "WordCount 1 MiB Zipf text, V=10k", 1),
    "C2": ("sm", "StringMatch 4 GiB text, 16-byte pattern", 4096),
    "C3": ("km", "KMeans one Lloyd step, 64M x 8 fp32, k=32", 64 << 20),
    "C4": ("ii", "InvertedIndex 8 GiB HTML-like", 8192),
    "C5": ("wc", "WordCount 8 GiB/GPU Zipf text, V=1M (weak)", 8192),
}


# BASELINE.json's metric (both arms print it, so the driver can divide them)
METRIC = "Map+Group+Reduce input GB/s and % HBM roofline at 1/2/4/8 B200 vs CPU oracle"
# strong scaling: total units of the whole job (C5: 64 GiB, configs[4]) and units per mapped batch
STRONG_TOTAL = {"C1": 1, "C2": 4096, "C3": 64 << 20, "C4": 8192, "C5": 65536}
BATCH_UNITS = {"C5": 8192}


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


def spec_for(cfg):
    from gen import pygen
    if cfg == "C1":
        return pygen.spec_wc(10_000, 1)
    if cfg == "C2":
        return pygen.spec_sm(1000, 2)
    if cfg == "C4":
        return pygen.spec_ii(4)
    if cfg == "C5":
        return pygen.spec_wc(1_000_000, 5)
    return pygen.KMSpec()


# ------------------------------------------------------------------ clocks (NVML, during timing)
class ClockSampler:
    REASONS = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x2: "applications_clocks_setting"}

    def __init__(self, dev):
        self.samples, self.reasons, self.stop_ev = [], set(), threading.Event()
        self.max_mhz = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(dev)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None
        self.t = threading.Thread(target=self._run, daemon=True)

    def _run(self):
        while not self.stop_ev.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.05)

    def __enter__(self):
        if self.nv:
            self.t.start()
        return self

    def __exit__(self, *a):
        self.stop_ev.set()
        if self.nv:
            self.t.join()

    def summary(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ------------------------------------------------------------------ inputs
def make_batches(cfg, u0, units, dev):
    """Device-resident synthetic input of global units [u0, u0 + units), as mapped batches of at
    most BATCH_UNITS[cfg] units (weak scaling: u0 = rank * P; strong: the rank's slice of the
    fixed total)."""
    from gen import pygen
    wl = WORKLOADS[cfg][0]
    spec = spec_for(cfg)
    step = BATCH_UNITS.get(cfg, units) or 1
    out = []
    for a in range(u0, u0 + units, step):
        m = min(step, u0 + units - a)
        if wl == "km":
            pts = pygen.device_km(spec, m, i0=a, device=dev)
            _, init = pygen.km_centres(spec)
            out.append({"wl": wl, "data": pts.view(-1).view(__import__("torch").uint8), "offsets": None, "n": m,
                        "nbytes": m * 32, "centroids": init, "spec": spec, "page0": a, "base": 0})
        else:
            g = pygen.device_text(spec, m, page0=a, device=dev)
            out.append({"wl": wl, "data": g["data"], "offsets": g["offsets"], "n": g["n"],
                        "nbytes": m * spec.page_bytes, "spec": spec, "page0": a, "base": g["base"]})
    return out


def job_kwargs(inp, flags=0, device=0, rank=0, world=1):
    kw = {"device": device, "flags": flags, "rank": rank, "nranks": world}
    if inp["wl"] == "sm":
        kw["pattern"] = inp["spec"].pattern
    if inp["wl"] == "km":
        kw["centroids"] = inp["centroids"]
    if inp["wl"] in ("sm", "ii"):
        kw["input_base"] = inp.get("base", 0)
    return kw


# ------------------------------------------------------------------ CPU oracle (baseline / reference arm)
def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    import platform
    return platform.processor() or "unknown"


def oracle_sample(cfg, sample_units, page0=0):
    """Time the oracle (as it stands; SURVEY §8(d) D-5 build: -O3 -march=native -ffp-contract=off,
    compiled on this host) on the first `sample_units` pages/points of rank 0's shard."""
    from gen import pygen
    from oracle import oracle
    oracle.use_native()
    wl = WORKLOADS[cfg][0]
    spec = spec_for(cfg)
    if wl == "km":
        pts = pygen.host_km(spec, sample_units, i0=page0)
        _, init = pygen.km_centres(spec)
        data = pts.view(np.uint8).reshape(-1)
        t0 = time.perf_counter()
        oracle.run("km", [(data, None, sample_units, 32, 0)], centroids=init)
        dt = time.perf_counter() - t0
        return data.size, dt, f"first {sample_units} points ({data.size / 2**20:.0f} MiB) of the shard"
    g = pygen.host_text(spec, sample_units, page0=page0)
    kw = {"pattern": spec.pattern} if wl == "sm" else {}
    t0 = time.perf_counter()
    oracle.run(wl, [(g["data"], g["offsets"], g["n"], 0, g["base"])], **kw)
    dt = time.perf_counter() - t0
    return g["data"].size, dt, f"first {sample_units} pages ({sample_units} MiB) of the shard"


def cpu_info():
    from oracle import oracle
    return {"cores": 1, "cpu_model": cpu_model(), "oracle_build": oracle.build_flags(),
            "host_cores_available": len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else os.cpu_count()}


ORACLE_SAMPLE = {"C1": 1, "C2": 2048, "C3": 16 << 20, "C4": 2048, "C5": 96}   # ~10-30 s of CPU work
REF_STEP_SAMPLE = {"C1": 1, "C2": 4, "C3": 1 << 19, "C4": 8, "C5": 8}     # per reference-arm step


def run_reference(args, rank, world):
    if rank != 0:
        return
    cfg = args.workload
    su = REF_STEP_SAMPLE[cfg]
    for _ in range(args.warmup):
        oracle_sample(cfg, su)
    times = []
    nb = 0
    desc = ""
    for _ in range(args.steps):
        nb, dt, desc = oracle_sample(cfg, su)
        times.append(dt)
    ms = 1000.0 * sum(times) / len(times)
    val = nb / (ms / 1000.0) / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": round(val, 6),
            "unit": "GB/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(ms, 3), "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None,
            "dtype": "u8" if WORKLOADS[cfg][0] != "km" else "f32", "data": "synthetic",
            "config": {"workload": cfg, "description": WORKLOADS[cfg][1], "sample": desc,
                       "parallelism": f"dp{world}"},
            "cpu_baseline": {"value": round(val, 6), "unit": "GB/s", "kind": "oracle", "sample": desc, **cpu_info()},
            "e2e": {"value": round(val, 6), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ GPU arm
def algorithmic(inp, st, steps):
    """Algorithmic bytes per step of each phase.

    WordCount Map output is three streams: exact keys (words <= 5 bytes) are bare 4-B u32 keys
    sorted keys-only (4 B read + 4 B written per pass); mid keys (6..8 bytes) bare 8-B keys
    (8 B read + 8 B written per pass); hashed keys
    (longer words) carry a key reference (16 B) and sort with a u32 permutation (24 B per pass,
    the first pass reads no permutation)."""
    wl = inp["wl"]
    m = st["pairs"] / steps
    mh = st["pairs_hashed"] / steps
    mc = st["pairs_mid"] / steps
    mx = m - mh - mc
    n = inp["n"]
    off_b = 8 * (n + 1) if inp["offsets"] is not None else 0
    px = st["sort_passes_keys"] / steps
    pc = st["sort_passes_mid"] / steps
    passes = st["sort_passes"] / steps
    if wl == "wc":
        map_b = inp["nbytes"] + off_b + mx * 4 + mc * 8 + mh * 16
        ph = passes - px - pc
        sort_b = px * 8 * mx + pc * 16 * mc + ((ph * 24 - 4) * mh if ph else 0.0)
    else:
        if wl == "sm":   # lazy record directory: offsets are read only around pattern candidates
            off_b = 0
        if wl == "km" and st.get("words_combined", 0):   # KM combiner: no pairs written
            map_b = inp["nbytes"]
        else:
            map_b = inp["nbytes"] + off_b + m * {"sm": 8, "km": 40, "ii": 24}[wl]
        sort_b = (passes * 24 - 4) * m if passes else 0.0   # first pass reads no payload
    hist_b = (4 * mx + 8 * (mc + mh)) if wl == "wc" else 8 * m
    return {"map": map_b, "hist": hist_b, "sort": sort_b, "passes": passes, "pairs": m, "pairs_exact": mx,
            "passes_keys": px}


def relaunch(args_n):
    """--gpus N without a torchrun environment: run this script under torch.distributed.run with
    N ranks on this node (127.0.0.1 rendezvous); rank 0 prints the JSON line."""
    import socket
    import subprocess
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args_n}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="C5", choices=sorted(WORKLOADS))
    ap.add_argument("--impl", default="bmr", choices=["bmr", "reference"])
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="weak: the 1-GPU shard per GPU; strong: fixed total (C5 64 GiB) split over the GPUs")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--units", type=int, default=0, help="override pages (text) / points (KM) per GPU")
    ap.add_argument("--mode", default="SIO", choices=["SIO", "SO", "SI", "G"],
                    help="Map memory-usage mode (PAPER.md L129-135 ablation, SURVEY §8(f) f-2)")
    ap.add_argument("--no-map-combine", action="store_true", help="literal north-star order (no Map combiner)")
    ap.add_argument("--km-full-scan", action="store_true",
                    help="KMeans: every point scans all k centroids (no bound test; the paper's literal Map)")
    ap.add_argument("--xchg", default="nccl", choices=["nccl", "caller", "fused"],
                    help="exchange at N > 1: libbmr's mr_group over NCCL (nccl), torch.distributed moving the "
                         "partition buffers (caller), or the fused Map flush into receive windows (fused, II)")
    args = ap.parse_args()

    env_world = os.environ.get("WORLD_SIZE")
    if env_world is None and args.gpus > 1:
        sys.exit(relaunch(args.gpus))
    world = int(env_world or "1")
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus and rank == 0:
        sys.stderr.write(f"[bench] --gpus {args.gpus} but WORLD_SIZE={world}: using the launched world\n")
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    share = os.environ.get("BMR_SHARE_GPU") == "1" and world > 1
    if share:   # plumbing test on a 1-GPU box: every rank on cuda:0, each its own NCCL "host"
        local = 0
        os.environ.setdefault("NCCL_HOSTID", f"bmrbench{rank}")
        os.environ.setdefault("NCCL_SOCKET_IFNAME", "lo")
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_jim11_b200 as bmr

    torch.cuda.set_device(local)
    dev = f"cuda:{local}"
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device(dev))

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    cfg = args.workload
    wl = WORKLOADS[cfg][0]
    if args.units:
        w = WORKLOADS[cfg]
        WORKLOADS[cfg] = (w[0], w[1] + f" [reduced: {args.units} units]", args.units)
    P = WORKLOADS[cfg][2]
    if args.scaling == "strong":
        T = args.units or STRONG_TOTAL[cfg]
        u0, units = rank * T // world, (rank + 1) * T // world - rank * T // world
    else:
        u0, units = rank * P, P
    batches = make_batches(cfg, u0, units, dev)
    inp = batches[0]
    nbytes_rank = sum(b["nbytes"] for b in batches)
    n_rank = sum(b["n"] for b in batches)
    torch.cuda.synchronize()
    mode_flags = {"SIO": 0, "SO": bmr.FLAG_NO_SMEM_IN, "SI": bmr.FLAG_NO_SMEM_OUT,
                  "G": bmr.FLAG_NO_SMEM_IN | bmr.FLAG_NO_SMEM_OUT}[args.mode]
    if args.no_map_combine:
        mode_flags |= bmr.FLAG_NO_MAP_COMBINE
    if args.km_full_scan:
        mode_flags |= bmr.FLAG_KM_FULL_SCAN
    if len(batches) > 1 and wl == "wc":
        mode_flags |= bmr.FLAG_BATCH_COMBINE   # per-batch group + combine (SURVEY §8(e) strong scaling)
    exchange = world > 1 and wl != "sm"       # SM is Map-only: no exchange
    comm = bmr.Comm.from_torch() if exchange and args.xchg == "nccl" else None
    job = bmr.Job(wl, comm=comm, **job_kwargs(inp, bmr.FLAG_PROFILE | mode_flags, local, rank, world))
    stream = torch.cuda.current_stream()
    xwin = None
    if args.xchg == "fused" and world >= 1 and wl == "ii":
        # every rank's receive window holds what all ranks may send it (uniform hash partition;
        # 2x headroom for skew)
        ecap = 2 * nbytes_rank // 48 + 4096
        hcap = 2 * nbytes_rank // 4 + 65536
        if world > 1:   # windows shared through CUDA IPC: the Maps store into peers over NVLink
            from paper_conf_ipps_jim11_b200 import dist as D
            xwin = bmr.XWindow(ecap, hcap, device=torch.device(dev), ipc=True)
            job.set_xwindows(D.open_xwindows(xwin))
        else:
            xwin = bmr.XWindow(ecap, hcap, device=torch.device(dev))
            job.set_xwindows([xwin])
        exchange = False
    elif args.xchg == "fused":
        raise SystemExit("--xchg fused: InvertedIndex only")

    def step():
        job.reset()
        if xwin is not None:   # f-3: the Maps append the records to the owners' windows, then ingest
            xwin.reset()
            barrier()          # every window is empty before any rank maps
            for b in batches:
                job.map(b["data"], b["offsets"], b["n"])
            barrier()          # every rank's records have landed
            job.ingest_xwindow(xwin)
        else:
            for b in batches:
                job.map(b["data"], b["offsets"], b["n"])
        if exchange and args.xchg == "caller":   # torch.distributed moves the partition buffers
            job.shuffle()
        job.group()            # (--xchg nccl: the exchange happens inside mr_group)
        job.reduce()

    for _ in range(max(3, args.warmup)):
        step()
    job.fetch()
    barrier()
    job.reset()
    # timed region: K steps, per-phase device times from the job's CUDA events
    acc = {k: 0.0 for k in ("map_ms", "hist_ms", "sort_ms", "seg_ms", "sort_keys_ms", "xchg_ms")}
    tot = {"pairs": 0, "sort_passes": 0, "kernel_launches": 0, "flushes": 0, "n_keys": 0, "pairs_hashed": 0,
           "sort_passes_keys": 0, "pairs_mid": 0, "sort_passes_mid": 0, "words_combined": 0, "pairs_partial": 0,
           "collisions": 0, "xchg_send_bytes": 0, "replays": 0, "map_seal_waits": 0, "map_spills": 0,
           "km_points_scanned": 0}
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        barrier()
        t0 = time.perf_counter()
        ev0.record(stream)
        evs = []
        for _ in range(args.steps):
            step()
            e = torch.cuda.Event(enable_timing=True)
            e.record(stream)
            evs.append(e)
            st = job.stats()  # map/hist/sort/seg events are collected at mr_group's synchronisation
            for k in tot:
                tot[k] += st[k]
            for k in acc:
                acc[k] += st[k]
        ev1.record(stream)
        ev1.synchronize()
        wall = time.perf_counter() - t0
        barrier()
    ms = ev0.elapsed_time(ev1) / args.steps
    step_ms = [ev0.elapsed_time(evs[0])] + [evs[i - 1].elapsed_time(evs[i]) for i in range(1, len(evs))]
    t = torch.tensor([ms], device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max = float(t.item())
    # reduce-phase events are collected at mr_fetch: one extra (untimed) pass of K steps
    red = 0.0
    for _ in range(args.steps):
        step()
        job.fetch()
        red += job.stats()["reduce_ms"]
    per = {k: v / args.steps for k, v in acc.items()}
    per["reduce_ms"] = red / args.steps
    alg = algorithmic(dict(inp, n=n_rank, nbytes=nbytes_rank), tot, args.steps)
    hbm, peak_kind = load_peaks()
    # roofline of the dominant kernel (the larger device-time share of the step): the Map kernel
    # or the onesweep LSD passes (all sort streams together, per launch)
    map_ach = alg["map"] / (per["map_ms"] / 1e3) / 1e9 if per["map_ms"] else 0.0
    sort_ms_all = per["sort_ms"]
    if alg["passes"] and sort_ms_all > per["map_ms"]:
        if alg["passes_keys"] and per["sort_keys_ms"] > 0.5 * sort_ms_all:
            kname = "k_onesweep (keys-only u32 LSD pass, WC exact stream)"
            launch_ms = per["sort_keys_ms"] / alg["passes_keys"]
            launch_bytes = 8 * alg["pairs_exact"]
        else:
            kname = "k_onesweep (LSD pass)"
            launch_ms = sort_ms_all / alg["passes"]
            launch_bytes = alg["sort"] / alg["passes"]
        tkey = "k_onesweep"
    else:
        kname, launch_ms, launch_bytes, tkey = "k_map", per["map_ms"], alg["map"], "k_map"
    nmaps = len(batches)
    if tkey == "k_map" and nmaps > 1:   # one Map launch per batch
        launch_ms, launch_bytes = launch_ms / nmaps, launch_bytes / nmaps
    ach = launch_bytes / (launch_ms / 1e3) / 1e9 if launch_ms else 0.0
    roof = {"kernel": kname, "bound": "hbm", "achieved": round(ach, 1), "peak": hbm, "peak_kind": peak_kind,
            "unit": "GB/s", "frac": round(ach / hbm, 4), "traffic": None, "bytes_per_launch": int(launch_bytes),
            "ms_per_launch": round(launch_ms, 4),
            "share_of_step": round((sort_ms_all if tkey == "k_onesweep" else per["map_ms"]) / ms, 3)}
    km_stats = None
    if wl == "km" and tkey == "k_map":
        # KMeans Map.  Full scan (--km-full-scan): FP32-pipe bound, per point k
        # centroids x 8 dims x (sub + fma) lane-ops against 148 SMs x 128 FP32 lanes x the max SM
        # clock.  Default (bound test): a shortcut point costs one centroid (16
        # lane-ops), so the Map is bound by its HBM read; the FP32 figure is then reported on the
        # lane-ops actually executed.
        k = len(inp["centroids"])
        scanned = tot["km_points_scanned"] / args.steps / nmaps
        pts_launch = n_rank / nmaps
        full = bool(args.km_full_scan) or scanned >= pts_launch
        ops_exec = 16.0 * k * scanned + 16.0 * (pts_launch - scanned)
        ops = 16.0 * k * pts_launch if full else ops_exec
        clk_mhz = 1965.0
        try:
            clk_mhz = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["sm_max_mhz"])
        except Exception:
            pass
        peak_ops = 148 * 128 * clk_mhz * 1e6
        fp32 = {"achieved": round(ops / (launch_ms / 1e3) / 1e12, 3), "peak": round(peak_ops / 1e12, 2),
                "peak_kind": f"derived: 148 SMs x 128 FP32 lanes x {clk_mhz:.0f} MHz (FFMA/FFMA2, fma pipe)",
                "unit": "Tlane-op/s", "frac": round(ops / (launch_ms / 1e3) / peak_ops, 4),
                "ops_per_launch": int(ops), "ops_basis": "all k centroids per point" if full else
                "executed: k centroids per scanned point, 1 per bound-test point"}
        km_stats = {"full_scan": bool(args.km_full_scan), "points_scanned_per_launch": int(scanned),
                    "bound_test_frac": round(1.0 - scanned / pts_launch, 6) if pts_launch else None}
        if full:
            roof_hbm = dict(roof)
            roof = {"kernel": "k_map (KMeans distances)", "bound": "fp32", **{k2: fp32[k2] for k2 in (
                "achieved", "peak", "peak_kind", "unit", "frac", "ops_per_launch")}, "traffic": None,
                    "ms_per_launch": round(launch_ms, 4), "share_of_step": roof["share_of_step"],
                    "hbm": {k2: roof_hbm[k2] for k2 in ("achieved", "peak", "frac")}}
        else:
            roof["kernel"] = "k_map (KMeans, bound test)"
            roof["fp32"] = fp32
    traffic_p = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(traffic_p):
        tr = json.load(open(traffic_p)).get(cfg, {}).get(tkey)
        if tr:
            roof["traffic"] = tr["bytes_per_launch"]
            roof["traffic_source"] = tr["source"]

    nbytes_all = nbytes_rank * world if args.scaling == "weak" else (args.units or STRONG_TOTAL[cfg]) * (
        32 if wl == "km" else inp["spec"].page_bytes)
    value = nbytes_all / (ms_max / 1e3) / 1e9

    # ---- end to end: host buffers through mr_map_host(_lines), H2D + D2H inside the timed region
    e2e = None
    if args.e2e_steps > 0 and len(batches) == 1 and xwin is None:
        h_data = torch.empty(inp["data"].numel(), dtype=torch.uint8, pin_memory=True)
        h_data.copy_(inp["data"])
        h_off = inp["offsets"]   # text workloads: only a flag here (offsets are derived on the device)
        torch.cuda.synchronize()
        job_e = bmr.Job(wl, comm=comm, **job_kwargs(inp, mode_flags, local, rank, world))
        d2h = 0

        def estep():
            job_e.reset()
            if h_off is None:   # KM: fixed-stride records
                job_e.map_host(h_data.numpy(), None, inp["n"])
            else:               # text: records are the lines; offsets derived on the device
                job_e.map_host_lines(h_data.numpy())
            if exchange and args.xchg == "caller":
                job_e.shuffle()
            job_e.group()
            job_e.reduce()
            r = job_e.fetch(copy=False)   # the D2H into job-owned pinned memory, no extra host copy
            return r["keys"].nbytes + r["vals"].nbytes + r["key_offsets"].nbytes + r["val_offsets"].nbytes

        estep()
        barrier()
        t0 = time.perf_counter()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.e2e_steps):
            d2h = estep()
        e1.record(stream)
        e1.synchronize()
        ems = max(e0.elapsed_time(e1), (time.perf_counter() - t0) * 1e3) / args.e2e_steps
        te = torch.tensor([ems], device=dev)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        ems = float(te.item())
        h2d = inp["nbytes"]   # text: the bytes only (mr_map_host_lines derives the offsets on the device)
        e2e = {"value": round(nbytes_all / (ems / 1e3) / 1e9, 3), "unit": "GB/s", "ms_per_step": round(ems, 3),
               "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
               "api": "mr_map_host_lines+mr_fetch" if h_off is not None else "mr_map_host+mr_fetch"}
        job_e.close()

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        su = ORACLE_SAMPLE[cfg]
        nb, dt, desc = oracle_sample(cfg, su)
        cpu = {"value": round(nb / dt / 1e9, 6), "unit": "GB/s", "kind": "oracle", "sample": desc,
               "seconds": round(dt, 2), **cpu_info()}

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(value, 3), "unit": "GB/s",
            "n_gpus": world, "steps": args.steps, "warmup": max(3, args.warmup), "ms_per_step": round(ms_max, 3),
            "us_per_step": round(ms_max * 1e3, 1),
            "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None,
            "dtype": "f32" if wl == "km" else "u8", "data": "synthetic",
            "config": {"workload": cfg, "description": WORKLOADS[cfg][1],
                       "input_bytes_per_gpu": nbytes_rank, "records_per_gpu": n_rank, "batches_per_gpu": nmaps,
                       "input_bytes_total": nbytes_all,
                       "l2": "inputs larger than L2 (no flush needed)" if nbytes_rank > (256 << 20) else
                             "input smaller than L2: L2-resident (C1 is reported in us)",
                       "parallelism": f"dp{world}", "map_mode": args.mode, "map_combiner": not args.no_map_combine,
                       **({"shared_gpu_plumbing_test": True} if share else {})},
            "records_per_s": round(n_rank * world / (ms_max / 1e3), 1),
            "hbm_frac_end_to_end": round((alg["map"] + alg["hist"] + alg["sort"]) / (ms_max / 1e3) / 1e9 / hbm, 4),
            "hbm_frac_nominal_8tbs": round((alg["map"] + alg["hist"] + alg["sort"]) / (ms_max / 1e3) / 1e9 / 8000.0, 4),
            "phases_ms": {k[:-3]: round(v, 3) for k, v in per.items()},
            "map": {"achieved_gbs": round(map_ach, 1), "frac": round(map_ach / hbm, 4),
                    "frac_nominal_8tbs": round(map_ach / 8000.0, 4), "bytes_per_step": int(alg["map"])},
            "pairs_per_step": int(alg["pairs"]), "sort_passes": alg["passes"],
            "wc_streams": ({"exact": int(alg["pairs_exact"]), "mid": int(tot["pairs_mid"] / args.steps),
                            "hashed": int(tot["pairs_hashed"] / args.steps),
                            "partials": int(tot["pairs_partial"] / args.steps)} if wl == "wc" else None),
            "map_combiner": {"words_or_points_absorbed": int(tot["words_combined"] / args.steps)},
            "distinct_keys": int(tot["n_keys"] / args.steps),
            "hash_collisions_per_step": tot["collisions"] / args.steps,
            "replays": tot["replays"],
            "map_output_ring": {"seal_waits_per_step": tot["map_seal_waits"] / args.steps,
                                "spills_per_step": tot["map_spills"] / args.steps},
            "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "kmeans": km_stats,
            "exchange": ({"kind": ("libbmr mr_group over NCCL (" + bmr.Comm.backend() + ")") if args.xchg == "nccl"
                          else "torch.distributed all_to_all_single (NCCL) of libbmr's partition buffers",
                          "ranks": world, "send_bytes_per_rank": int(tot["xchg_send_bytes"] / args.steps),
                          "xchg_ms": round(per["xchg_ms"], 3), "combiner": wl in ("wc", "km")} if exchange else
                         ({"kind": "fused Map flush into the owners' receive windows (f-3, CUDA IPC / NVLink)",
                           "window_entries_heap": list(xwin.used())} if xwin is not None else None)),
            "gpu_launches": int(tot["kernel_launches"]),
            "clocks": clk.summary(), "wall_s_timed": round(wall, 3),
            "step_ms": {"min": round(min(step_ms), 3), "median": round(statistics.median(step_ms), 3),
                        "max": round(max(step_ms), 3)},
        }
        print(json.dumps(line), flush=True)
    job.close()
    if comm is not None:
        comm.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
