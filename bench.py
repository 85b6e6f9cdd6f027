#!/usr/bin/env python
"""bench.py — libbmr hot-path benchmark (BASELINE.json metric: Map+Group+Reduce input GB/s and
% HBM roofline, vs the CPU oracle).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C5|C4|C3|C2|C1] [--impl reference]
                    [--mode SIO|SO|SI|G] [--no-map-combine] [--xchg a2a|fused] [--units U]

One step = one pass of the whole hot path (tile scheduling, stage-in,
user map, emit, flush, digit histogram, onesweep passes, segment boundaries, reduce + output
assembly) over one shard of synthetic input already resident in HBM.  Default workload = C5
(WordCount, Zipf V=1M, 8 GiB per GPU, weak scaling): the configuration the metric's
"1/2/4/8 B200" is quoted on that exercises every row (C2 StringMatch is Map-only).
Prints ONE JSON line on rank 0.  Timing: W warm-up steps, then K steps bracketed by barrier +
cuda.synchronize, CUDA events on the job stream, max over ranks.  Inputs (8 GiB) exceed L2
(126 MB), so no extra flush is needed.  At N > 1 the exchange is the partition + all-to-all over
NCCL, or with --xchg fused (InvertedIndex) the Maps store straight into the owners' receive
windows through CUDA IPC.
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
def make_input(cfg, rank, dev):
    """Device-resident synthetic shard of rank `rank` (weak scaling: global units r*P..)."""
    from gen import pygen
    wl, _, units = WORKLOADS[cfg]
    spec = spec_for(cfg)
    if wl == "km":
        pts = pygen.device_km(spec, units, i0=rank * units, device=dev)
        _, init = pygen.km_centres(spec)
        return {"wl": wl, "data": pts.view(-1).view(__import__("torch").uint8), "offsets": None, "n": units,
                "nbytes": units * 32, "centroids": init, "spec": spec, "page0": rank * units}
    g = pygen.device_text(spec, units, page0=rank * units, device=dev)
    return {"wl": wl, "data": g["data"], "offsets": g["offsets"], "n": g["n"], "nbytes": units * spec.page_bytes,
            "spec": spec, "page0": rank * units, "base": g["base"]}


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
def oracle_sample(cfg, sample_units, page0=0):
    """Time the oracle (as it stands) on the first `sample_units` pages/points of rank 0's shard."""
    from gen import pygen
    from oracle import oracle
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
    line = {"impl": "reference", "metric": "Map+Group+Reduce input GB/s (CPU oracle)", "value": round(val, 6),
            "unit": "GB/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(ms, 3), "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "u8" if WORKLOADS[cfg][0] != "km" else "f32", "data": "synthetic",
            "config": {"workload": cfg, "description": WORKLOADS[cfg][1], "sample": desc},
            "cpu_baseline": {"value": round(val, 6), "unit": "GB/s", "cores": 1, "kind": "oracle", "sample": desc},
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="C5", choices=sorted(WORKLOADS))
    ap.add_argument("--impl", default="bmr", choices=["bmr", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--units", type=int, default=0, help="override pages (text) / points (KM) per GPU")
    ap.add_argument("--mode", default="SIO", choices=["SIO", "SO", "SI", "G"],
                    help="Map memory-usage mode (PAPER.md L129-135 ablation, SURVEY §8(f) f-2)")
    ap.add_argument("--no-map-combine", action="store_true", help="literal north-star order (no Map combiner)")
    ap.add_argument("--xchg", default="a2a", choices=["a2a", "fused"],
                    help="InvertedIndex exchange: partition + all-to-all (a2a) or the fused Map flush into "
                         "receive windows (f-3; one GPU: the rank's own window, timed with its ingest)")
    args = ap.parse_args()

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

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

    if args.units:
        w = WORKLOADS[args.workload]
        WORKLOADS[args.workload] = (w[0], w[1] + f" [reduced: {args.units} units]", args.units)
    inp = make_input(args.workload, rank, dev)
    torch.cuda.synchronize()
    mode_flags = {"SIO": 0, "SO": bmr.FLAG_NO_SMEM_IN, "SI": bmr.FLAG_NO_SMEM_OUT,
                  "G": bmr.FLAG_NO_SMEM_IN | bmr.FLAG_NO_SMEM_OUT}[args.mode]
    if args.no_map_combine:
        mode_flags |= bmr.FLAG_NO_MAP_COMBINE
    job = bmr.Job(inp["wl"], **job_kwargs(inp, bmr.FLAG_PROFILE | mode_flags, local, rank, world))
    stream = torch.cuda.current_stream()
    exchange = world > 1 and inp["wl"] != "sm"      # SM is Map-only: no exchange
    xbytes = [0]
    xwin = None
    if args.xchg == "fused":
        if inp["wl"] != "ii":
            raise SystemExit("--xchg fused: InvertedIndex only")
        # every rank's receive window holds what all ranks may send it (uniform hash partition;
        # 2x headroom for skew)
        ecap = 2 * inp["nbytes"] // 48 + 4096
        hcap = 2 * inp["nbytes"] // 4 + 65536
        if world > 1:   # windows shared through CUDA IPC: the Maps store into peers over NVLink
            from paper_conf_ipps_jim11_b200 import dist as D
            xwin = bmr.XWindow(ecap, hcap, device=torch.device(dev), ipc=True)
            job.set_xwindows(D.open_xwindows(xwin))
        else:
            xwin = bmr.XWindow(ecap, hcap, device=torch.device(dev))
            job.set_xwindows([xwin])
        exchange = False

    def step():
        job.reset()
        if xwin is not None:   # f-3: the Maps append the records to the owners' windows, then ingest
            xwin.reset()
            barrier()          # every window is empty before any rank maps
            job.map(inp["data"], inp["offsets"], inp["n"])
            barrier()          # every rank's records have landed
            job.ingest_xwindow(xwin)
        else:
            job.map(inp["data"], inp["offsets"], inp["n"])
        if exchange:  # one hash all-to-all over NCCL
            xbytes[0] = job.shuffle()
        job.group()
        job.reduce()

    for _ in range(max(3, args.warmup)):
        step()
    job.fetch()
    barrier()
    job.reset()
    # timed region: K steps, per-phase device times from the job's CUDA events
    acc = {k: 0.0 for k in ("map_ms", "hist_ms", "sort_ms", "seg_ms", "sort_keys_ms")}
    tot = {"pairs": 0, "sort_passes": 0, "kernel_launches": 0, "flushes": 0, "n_keys": 0, "pairs_hashed": 0,
           "sort_passes_keys": 0, "pairs_mid": 0, "sort_passes_mid": 0, "words_combined": 0, "pairs_partial": 0}
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
            s = job.stats()  # map/hist/sort/seg events are collected at mr_group's synchronisation
            for k in tot:
                tot[k] += s[k]
            for k in acc:
                acc[k] += s[k]
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
    alg = algorithmic(inp, tot, args.steps)
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
    ach = launch_bytes / (launch_ms / 1e3) / 1e9 if launch_ms else 0.0
    roof = {"kernel": kname, "bound": "hbm", "achieved": round(ach, 1), "peak": hbm, "peak_kind": peak_kind,
            "unit": "GB/s", "frac": round(ach / hbm, 4), "traffic": None, "bytes_per_launch": int(launch_bytes),
            "ms_per_launch": round(launch_ms, 4),
            "share_of_step": round((sort_ms_all if tkey == "k_onesweep" else per["map_ms"]) / ms, 3)}
    traffic_p = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(traffic_p):
        tr = json.load(open(traffic_p)).get(args.workload, {}).get(tkey)
        if tr:
            roof["traffic"] = tr["bytes_per_launch"]
            roof["traffic_source"] = tr["source"]

    nbytes_all = inp["nbytes"] * world
    value = nbytes_all / (ms_max / 1e3) / 1e9

    # ---- end to end: host buffers through mr_map_host, H2D + D2H inside the timed region
    e2e = None
    if args.e2e_steps > 0:
        h_data = torch.empty(inp["data"].numel(), dtype=torch.uint8, pin_memory=True)
        h_data.copy_(inp["data"])
        h_off = inp["offsets"]   # text workloads: only a flag here (offsets are derived on the device)
        torch.cuda.synchronize()
        job_e = bmr.Job(inp["wl"], **job_kwargs(inp, mode_flags, local, rank, world))
        d2h = 0

        def estep():
            job_e.reset()
            if h_off is None:   # KM: fixed-stride records
                job_e.map_host(h_data.numpy(), None, inp["n"])
            else:               # text: records are the lines; offsets derived on the device
                job_e.map_host_lines(h_data.numpy())
            if exchange:
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
        su = ORACLE_SAMPLE[args.workload]
        nb, dt, desc = oracle_sample(args.workload, su)
        cpu = {"value": round(nb / dt / 1e9, 6), "unit": "GB/s", "cores": 1, "kind": "oracle", "sample": desc,
               "seconds": round(dt, 2)}

    if rank == 0:
        wl = inp["wl"]
        line = {
            "metric": "Map+Group+Reduce input GB/s", "value": round(value, 3), "unit": "GB/s",
            "n_gpus": world, "steps": args.steps, "warmup": max(3, args.warmup), "ms_per_step": round(ms_max, 3),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "f32" if wl == "km" else "u8", "data": "synthetic",
            "config": {"workload": args.workload, "description": WORKLOADS[args.workload][1],
                       "input_bytes_per_gpu": inp["nbytes"], "records_per_gpu": inp["n"],
                       "l2": "inputs larger than L2 (no flush needed)", "parallelism": f"dp{world}",
                       "map_mode": args.mode, "map_combiner": not args.no_map_combine},
            "records_per_s": round(inp["n"] * world / (ms_max / 1e3), 1),
            "hbm_frac_end_to_end": round((alg["map"] + alg["hist"] + alg["sort"]) / (ms_max / 1e3) / 1e9 / hbm, 4),
            "phases_ms": {k[:-3]: round(v, 3) for k, v in per.items()},
            "map": {"achieved_gbs": round(map_ach, 1), "frac": round(map_ach / hbm, 4),
                    "bytes_per_step": int(alg["map"])},
            "pairs_per_step": int(alg["pairs"]), "sort_passes": alg["passes"],
            "wc_streams": ({"exact": int(alg["pairs_exact"]), "mid": int(tot["pairs_mid"] / args.steps),
                            "hashed": int(tot["pairs_hashed"] / args.steps),
                            "partials": int(tot["pairs_partial"] / args.steps)} if inp["wl"] == "wc" else None),
            "map_combiner": {"words_or_points_absorbed": int(tot["words_combined"] / args.steps)},
            "distinct_keys": int(tot["n_keys"] / args.steps),
            "roofline": roof, "cpu_baseline": cpu, "e2e": e2e,
            "exchange": ({"kind": "hash all-to-all over NCCL (torch.distributed)", "send_bytes_per_rank": xbytes[0],
                          "combiner": inp["wl"] in ("wc", "km")} if exchange else
                         ({"kind": "fused Map flush into the owners' receive windows (f-3, CUDA IPC / NVLink)",
                           "window_entries_heap": list(xwin.used())} if xwin is not None else None)),
            "gpu_launches": int(tot["kernel_launches"]),
            "clocks": clk.summary(), "wall_s_timed": round(wall, 3),
            "step_ms": {"min": round(min(step_ms), 3), "median": round(statistics.median(step_ms), 3),
                        "max": round(max(step_ms), 3)},
        }
        print(json.dumps(line), flush=True)
    job.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
