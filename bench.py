#!/usr/bin/env python
"""SNICIT hot-path benchmark: SDGC inference edges/s on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl snicit|reference]

A step = one whole SNICIT inference (all SURVEY 8(a) rows: pre-convergence layers, conversion,
post-convergence layers, recovery, categories) over one batch.  N=1 workload: config C2 (SDGC 4096
neurons x 480 layers, batch 60,000, t=30, s=32, n=16, eta=eps=0.03), synthetic inputs (DESIGN.md
section 5).  N>1 (torchrun, one rank per GPU, NCCL): weak scaling -- every rank infers its own 60,000-row
batch (global row ids offset by rank), the category ids are all-gathered; value = rows of all ranks x
connections / max-over-ranks step time.

value: device-resident inputs (Y0 already in HBM), CUDA events around exactly K steps on the stream the
library launches on, barrier + synchronize on both sides.  Inputs (983 MB) are larger than L2 (126 MB), so
no explicit L2 flush.  e2e: the same metric through the C ABI with host (pinned) buffers: H2D of Y0 and D2H
of Y(L) + categories inside the timed region.

--impl reference: the CPU oracle (plain Eq. 1, oracle/) timed on the host cores on a bounded row sample of
the same workload (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from workload import sdgc  # noqa: E402

METRIC = "SDGC inference edges/sec at 1/2/4/8 B200; % of HBM roofline"
UNIT = "edges/s"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=5)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", choices=["snicit", "reference"], default="snicit")
    p.add_argument("--config", default="C2", choices=["C1", "C2", "C3", "C4", "C5"])
    p.add_argument("--mode", default="radix", choices=["radix", "perm", "random"])
    p.add_argument("--t", type=int, default=None)
    p.add_argument("--s", type=int, default=None)
    p.add_argument("--kernel", default="auto", choices=["auto", "ell", "circ"])
    p.add_argument("--load", default="auto", choices=["auto", "csc", "compact"],
                   help="network ABI: explicit CSC (snicit_load_network) or compact circulant form; auto = "
                        "compact for radix nets with N >= 16384 (C3/C4 CSC is 8-32 GB)")
    p.add_argument("--scaling", default="weak", choices=["weak", "strong"])
    p.add_argument("--batch", type=int, default=None, help="override rows per rank (weak) / global (strong)")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-uncompressed", action="store_true")
    p.add_argument("--pre-fused", type=int, default=1, choices=[0, 1, 2],
                   help="options.pre_fused: 1 = row-resident pre phase (default), 2 = without the constant-row "
                        "shortcut, 0 = one launch per layer")
    p.add_argument("--no-variants", action="store_true", help="skip the pre_fused = 2 / 0 roofline variants")
    p.add_argument("--cpu-seconds", type=float, default=15.0, help="target CPU work of the oracle sample")
    return p.parse_args()


def config_params(args):
    c = dict(sdgc.CONFIGS[args.config])
    if args.config == "C5":
        snic = dict(t=sdgc.medium_t(c["L"]), s=128, n=0)
    else:
        snic = dict(t=30, s=32, n=16)
    if args.t is not None:
        snic["t"] = args.t
    if args.s is not None:
        snic["s"] = args.s
    if args.batch is not None:
        c["B"] = args.batch
    return c, snic


def use_compact(args, c):
    if args.config == "C5" or args.mode != "radix":
        return False
    return args.load == "compact" or (args.load == "auto" and c["N"] >= 16384)


def make_network(args, c):
    if args.config == "C5":
        return sdgc.gen_medium_network(c["N"], c["L"])
    if use_compact(args, c):
        return sdgc.gen_circulant(c["N"], c["L"])
    return sdgc.gen_network(c["N"], c["L"], args.mode)


def oracle_layers(oracle, net, Y, nthreads=0):
    if isinstance(net, sdgc.CirculantNetwork):
        return oracle.layers_circulant_f32(net, Y, nthreads=nthreads)
    return oracle.layers_f32(net, Y, nthreads=nthreads)


def make_inputs(args, c, B, row0):
    if args.config == "C5":
        return sdgc.gen_medium_inputs(c["N"], B, row0=row0)
    return sdgc.gen_inputs(c["N"], B, row0=row0)


def cpu_info():
    model = ""
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return model


# ------------------------------------------------------------------ clocks (nvidia-smi during the timed region)
class ClockSampler:
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.th = threading.Thread(target=self._read, daemon=True)
            self.th.start()
        except (OSError, FileNotFoundError):
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return None
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, mx, reasons = [], 0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 8:
                continue
            try:
                sm.append(float(parts[0]))
                mx = max(mx, float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return None
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": len(sm)}


def committed_traffic(config: str):
    """Mean DRAM bytes per a1 layer-kernel launch from the latest committed ncu capture of this config
    (profiles/rNN_traffic_<config>.json, written by scripts/traffic.py), or (None, None)."""
    import glob
    files = sorted(glob.glob(os.path.join(os.path.dirname(os.path.abspath(__file__)), "profiles",
                                          f"r*_traffic_{config}.json")))
    if not files:
        return None, None
    d = json.load(open(files[-1]))
    return float(d["mean_dram_bytes_per_launch"]), f"{os.path.basename(files[-1])} ({d['launches']} launches)"


# FP32 FMA pipe of a B200: 148 SMs x 128 FMA lanes/clk x 2 flop x 1965 MHz (B200_PROFILING.md: 148 SMs,
# clocks.max.sm 1965 MHz; 128 FP32 lanes per SM: scripts/ubench_ffma.cu measured 127.9 FMA/clk/SM =
# 37.1 TFMA/s for FFMA and FFMA2 alike)
FMA_PEAK_TFLOPS = 148 * 128 * 2 * 1965e6 / 1e12
FMA_PEAK_SRC = ("derived: 148 SMs x 128 FP32 FMA/clk x 2 flop x 1965 MHz = 74.45 TFLOP/s (DESIGN.md §7; "
                "scripts/ubench_ffma.cu measured 74.2)")


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


def oracle_sample_time(oracle, net, Y, cores, seconds, probe_only=False, max_rows=None):
    """Rows of Y the oracle processes in ~`seconds` on all host cores (calibrated on `cores` rows run
    with all threads; at most `max_rows`, default len(Y)), and the measured time for that many rows."""
    cap = len(Y) if max_rows is None else max_rows
    # probe sizes double until one takes >= seconds / 2 (small probes are dominated by per-call and
    # thread start-up cost, which would under-size the sample)
    k = max(1, min(len(Y), cores))
    while True:
        t0 = time.perf_counter()
        oracle_layers(oracle, net, Y[:k])
        t_probe = max(time.perf_counter() - t0, 1e-6)
        if t_probe >= seconds / 2 or k >= len(Y):
            break
        k = min(len(Y), 2 * k)
    rows = int(max(k, min(cap, k * seconds / t_probe)))
    if probe_only:
        return rows, None
    if rows == k:
        return k, t_probe
    t0 = time.perf_counter()
    oracle_layers(oracle, net, Y[:rows])
    return rows, time.perf_counter() - t0


# ------------------------------------------------------------------ reference arm (CPU oracle)
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle

    c, snic = config_params(args)
    net = make_network(args, c)
    nnz = net.nnz
    cores = os.cpu_count() or 1
    # size the per-step sample to ~cpu_seconds / steps of the oracle on all cores
    probe = make_inputs(args, c, min(c["B"], 64 * cores), 0)
    rows, _ = oracle_sample_time(oracle, net, probe, cores, args.cpu_seconds / max(args.steps, 1), probe_only=True,
                                 max_rows=c["B"])
    Y = make_inputs(args, c, rows, 0)
    if args.warmup > 0:
        oracle_layers(oracle, net, Y[: max(1, min(rows, cores))])
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle_layers(oracle, net, Y)
        times.append(time.perf_counter() - t0)
    T = float(np.mean(times))
    value = rows * nnz / T
    sample = f"{rows} of {c['B']} rows of {args.config} (plain Eq. 1 oracle, all {net.L} layers), per step"
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": T * 1e3, "higher_is_better": True,
        "scaling": args.scaling, "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": f"{args.config}: {c['desc']}", "neurons": c["N"], "layers": c["L"],
                   "batch": c["B"], "w_mode": args.mode, "t": snic["t"], "s": snic["s"]},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample,
                         "cpu": cpu_info()},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ SNICIT arm
def run_snicit(args):
    import torch
    import torch.distributed as dist

    from paper_conf_icpp_jiangh0h23_b200 import KERNEL_AUTO, KERNEL_CIRC, KERNEL_ELL, SnicitNetwork, default_options
    from paper_conf_icpp_jiangh0h23_b200.parallel import allgather_categories, shard_rows

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    distributed = world > 1
    # SNICIT_DIST_BACKEND=gloo: test hook for boxes with fewer GPUs than ranks (ranks share devices,
    # collectives run on host tensors); the production path is NCCL, one rank per GPU
    backend = os.environ.get("SNICIT_DIST_BACKEND", "nccl")
    ndev = torch.cuda.device_count()
    dev = torch.device("cuda", local % max(ndev, 1))
    torch.cuda.set_device(dev)
    coll_dev = dev if backend == "nccl" else torch.device("cpu")
    if distributed:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)

    c, snic = config_params(args)
    if args.scaling == "weak":
        B_local, row0 = c["B"], rank * c["B"]
        B_global = c["B"] * world
    else:
        a, b = shard_rows(c["B"], world, rank)
        B_local, row0, B_global = b - a, a, c["B"]
    net = make_network(args, c)
    nnz = net.nnz
    kern = {"auto": KERNEL_AUTO, "ell": KERNEL_ELL, "circ": KERNEL_CIRC}[args.kernel]
    Yh = make_inputs(args, c, B_local, row0)
    if isinstance(net, sdgc.CirculantNetwork):
        g = SnicitNetwork.circulant(net.N, net.L, net.nu, net.w, net.bias, net.ymax, device=dev.index)
    else:
        g = SnicitNetwork.from_network(net, device=dev.index)
    stream = torch.cuda.Stream(device=dev)
    g.set_stream(stream)
    y0 = torch.from_numpy(Yh).to(dev)
    y_out = torch.empty_like(y0)
    opt = default_options(kernel=kern, n_segments=snic["n"], pre_fused=args.pre_fused)
    t, s = snic["t"], snic["s"]

    def step():
        g.infer(y0, t=t, s=s, options=opt, y_out=y_out, row_offset=row0)
        if distributed:
            with torch.cuda.stream(stream):
                ids = torch.from_numpy(g.categories()).to(coll_dev)
                allgather_categories(ids)
        else:
            g.num_categories()  # category set present (count read synchronises the stream)

    def timed(fn, k):
        if distributed:
            dist.barrier()
        torch.cuda.synchronize(dev)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(k):
            fn()
        e1.record(stream)
        torch.cuda.synchronize(dev)
        if distributed:
            dist.barrier()
        ms = e0.elapsed_time(e1) / k
        if distributed:
            tt = torch.tensor([ms], device=coll_dev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            ms = float(tt.item())
        return ms

    for _ in range(max(args.warmup, 3)):
        step()
    clocks = ClockSampler(local)
    clocks.start()
    ms = timed(step, args.steps)
    clk = clocks.stop()
    launches_per_step = g.stats()["kernel_launches"]
    value = B_global * nnz / (ms * 1e-3)

    # ---- roofline of the dominant kernel (the pre-convergence a1 kernel), live CUDA events
    def profile_pre(pre_fused):
        o = default_options(kernel=kern, n_segments=snic["n"], timing=2, pre_fused=pre_fused)
        g.infer(y0, t=t, s=s, options=o, y_out=y_out, row_offset=row0)  # first launches of these kernels
        pms, pbs = [], []
        for _ in range(max(1, min(args.steps, 3))):
            g.infer(y0, t=t, s=s, options=o, y_out=y_out, row_offset=row0)
            pr = g.layer_profile()
            pms.append(pr["ms"])
            pbs.append(pr["bytes"])
        st_ = g.stats()
        pm_ = np.mean(np.stack(pms), axis=0) if pms and len(pms[0]) else np.zeros(0)
        pb_ = pbs[0] if pbs else np.zeros(0)
        return st_, pm_, pb_

    st, pm, pb = profile_pre(args.pre_fused)
    phases = {k: st[k] for k in ("t_pre_ms", "t_convert_ms", "t_post_ms", "t_recover_ms", "t_total_ms")}
    peak, peak_src = measured_peaks()
    tag = args.config if args.t is None and args.mode == "radix" else None

    def hbm_roof(pm_, pb_, st_):
        """HBM roofline of the per-layer a1 kernels (8 B per live row-element per layer)."""
        avg_ms = float(pm_.mean())
        avg_bytes = float(pb_.mean())
        achieved = avg_bytes / (avg_ms * 1e-3) / 1e9
        traffic, traffic_src = committed_traffic(tag) if tag else (None, None)
        r = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
             "traffic": traffic, "traffic_unit": "bytes per launch (ncu dram read + write)",
             "traffic_source": traffic_src,
             "kernel": ("a1 layer kernels: layer_circ_kernel / layer_circ_seg_kernel (nu = 1), "
                        "layer_circ_col_kernel (strided)") if st_["circ_layers"] else "layer_ell_kernel",
             "peak_source": peak_src, "launches": int(len(pm_)), "avg_launch_ms": avg_ms,
             "avg_algorithmic_bytes": avg_bytes,
             "layer0_frac": float(pb_[0] / (pm_[0] * 1e-3) / 1e9 / peak)}
        if args.mode == "radix":  # per stride class (layer l has stride nu_l; DESIGN.md §7 kernels)
            strides = sdgc.radix_strides(c["N"])
            by = {}
            for l in range(len(pm_)):
                e = by.setdefault(f"nu={strides[l % len(strides)]}", [0, 0.0, 0.0])
                e[0] += 1
                e[1] += float(pm_[l])
                e[2] += float(pb_[l])
            r["by_stride"] = {k: {"launches": n, "ms": round(ms_, 4),
                                  "frac": round(b_ / (ms_ * 1e-3) / 1e9 / peak, 4)} for k, (n, ms_, b_) in by.items()}
        return r

    def alu_roof(pm_, pb_, st_):
        """FP32 FMA-pipe roofline of the row-resident kernel: algorithmic flops = 2 x 32 x N per full
        row-layer evaluation (constant rows carried by a scalar chain are not counted)."""
        kms = float(pm_.sum())
        flops = 2.0 * 32 * c["N"] * float(st_["pre_full_rows"])
        achieved = flops / (kms * 1e-3) / 1e12
        hbm_gbs = float(pb_.sum()) / (kms * 1e-3) / 1e9
        traffic, traffic_src = committed_traffic(tag + "_fused") if tag else (None, None)
        return {"bound": "alu", "achieved": achieved, "peak": FMA_PEAK_TFLOPS, "unit": "TFLOP/s",
                "frac": achieved / FMA_PEAK_TFLOPS, "traffic": traffic,
                "traffic_unit": "bytes per launch (ncu dram read + write)", "traffic_source": traffic_src,
                "kernel": "pre_fused_kernel (row-resident a1: layers 0..t-1 of a row in shared memory, FFMA2 chains)",
                "peak_source": FMA_PEAK_SRC, "launches": int(len(pm_)), "avg_launch_ms": kms,
                "algorithmic_flops": flops, "full_row_layers": int(st_["pre_full_rows"]),
                "const_rows": int(st_["pre_const_rows"]),
                "hbm": {"algorithmic_bytes": float(pb_.sum()), "achieved_gbs": hbm_gbs, "frac": hbm_gbs / peak}}

    roof = None
    if len(pm):
        roof = alu_roof(pm, pb, st) if st["pre_fused"] else hbm_roof(pm, pb, st)
        roof["share_of_step"] = float(pm.sum() / ms) if ms > 0 else None
        if st["pre_fused"] and ms > 0:
            # whole step: the step's algorithmic flops (the row-resident pre phase: post
            # layers of constant centroids are scalars) and bytes (pre phase + the live rows' final
            # activations written by the recovery) over the measured step time
            step_flops = roof["algorithmic_flops"]
            step_bytes = roof["hbm"]["algorithmic_bytes"] + 4.0 * c["N"] * st["live_at_t"]
            roof["whole_step"] = {"alu_frac": step_flops / (ms * 1e-3) / 1e12 / FMA_PEAK_TFLOPS,
                                  "hbm_frac": step_bytes / (ms * 1e-3) / 1e9 / peak,
                                  "algorithmic_flops": step_flops, "algorithmic_bytes": step_bytes}
        if st["pre_fused"] and not args.no_variants:
            # the same kernel with every live row evaluated in full (no constant-row shortcut), and the
            # per-layer kernels (one launch per layer, HBM-bound) on the same inputs
            st2, pm2, pb2 = profile_pre(2)
            if st2["pre_fused"] and len(pm2):
                r2 = alu_roof(pm2, pb2, st2)
                roof["no_const_skip"] = {k: r2[k] for k in ("achieved", "frac", "avg_launch_ms", "full_row_layers")}
            st0, pm0, pb0 = profile_pre(0)
            if len(pm0):
                r0 = hbm_roof(pm0, pb0, st0)
                roof["per_layer_kernels"] = {k: r0[k] for k in ("bound", "achieved", "peak", "unit", "frac", "traffic",
                                                                "traffic_source", "launches", "avg_launch_ms",
                                                                "by_stride") if k in r0}
                roof["per_layer_kernels"]["ms_total"] = float(pm0.sum())

    # ---- uncompressed GPU baseline (t >= L, same kernels)
    unc = None
    if not args.no_uncompressed:
        def step_unc():
            g.infer(y0, t=net.L, s=s, options=opt, y_out=y_out, row_offset=row0)
            g.num_categories()
        step_unc()
        ms_u = timed(step_unc, max(1, min(args.steps, 3)))
        unc = {"value": B_global * nnz / (ms_u * 1e-3), "unit": UNIT, "ms_per_step": ms_u,
               "speedup_snicit": ms_u / ms, "pre_fused": args.pre_fused}
        if args.pre_fused and not args.no_variants:  # plain layer-by-layer launches (no row residency)
            opt0 = default_options(kernel=kern, n_segments=snic["n"], pre_fused=0)

            def step_unc0():
                g.infer(y0, t=net.L, s=s, options=opt0, y_out=y_out, row_offset=row0)
                g.num_categories()
            step_unc0()
            ms_u0 = timed(step_unc0, max(1, min(args.steps, 3)))
            unc["per_layer_kernels"] = {"value": B_global * nnz / (ms_u0 * 1e-3), "ms_per_step": ms_u0}

    # ---- e2e through the C ABI with host (pinned) buffers.  Headline: the SDGC inputs are binary, so
    # Y0 is uploaded as the packed bitmap of snicit_infer_packed (H2D inside the call) and the step's
    # result is the category set (D2H).  Also reported: fp32 rows in and Y(L) out (e2e_fp32_io).
    e2e = e2e_fp32 = None
    if not args.no_e2e:
        from paper_conf_icpp_jiangh0h23_b200 import pack_rows
        binary = bool(np.all((Yh == 0) | (Yh == 1)))  # SDGC inputs; config 5's are real-valued
        bits_pin = torch.from_numpy(pack_rows(Yh if binary else Yh[:1] * 0).view(np.int32)).pin_memory()
        yh_pin = torch.from_numpy(Yh).pin_memory()
        yo_pin = torch.empty_like(yh_pin).pin_memory()

        def step_packed():
            g.infer_packed(bits_pin.numpy(), t=t, s=s, options=opt, row_offset=row0)
            cats = g.categories()
            if distributed:
                with torch.cuda.stream(stream):
                    allgather_categories(torch.from_numpy(cats).to(coll_dev))
            return cats

        def step_fp32():
            g.infer(yh_pin.numpy(), t=t, s=s, options=opt, y_out=yo_pin.numpy(), row_offset=row0)
            cats = g.categories()
            if distributed:
                with torch.cuda.stream(stream):
                    allgather_categories(torch.from_numpy(cats).to(coll_dev))
            return cats

        def wall(fn):
            fn()
            if distributed:
                dist.barrier()
            torch.cuda.synchronize(dev)
            k = max(1, min(args.steps, 3))
            t0 = time.perf_counter()
            for _ in range(k):
                cats = fn()
            torch.cuda.synchronize(dev)
            ms_e = (time.perf_counter() - t0) * 1e3 / k
            if distributed:
                tt = torch.tensor([ms_e], device=coll_dev)
                dist.all_reduce(tt, op=dist.ReduceOp.MAX)
                ms_e = float(tt.item())
            return ms_e, cats

        ms_f, cats = wall(step_fp32)
        e2e_fp32 = {"value": B_global * nnz / (ms_f * 1e-3), "unit": UNIT, "ms_per_step": ms_f,
                    "h2d_bytes_per_step": int(Yh.nbytes) * world, "d2h_bytes_per_step": (int(Yh.nbytes) + 8 * len(cats)) * world,
                    "api": "snicit_infer (fp32 Y0 in, fp32 Y(L) out) + snicit_categories",
                    "timer": "host wall clock around K synchronous C-ABI calls"}
        if binary:
            ms_e, cats = wall(step_packed)
            e2e = {"value": B_global * nnz / (ms_e * 1e-3), "unit": UNIT, "ms_per_step": ms_e,
                   "h2d_bytes_per_step": int(bits_pin.numel() * 4) * world, "d2h_bytes_per_step": (4 + 8 * len(cats)) * world,
                   "api": "snicit_infer_packed (Y0 as packed binary bitmap) + snicit_categories",
                   "timer": "host wall clock around K synchronous C-ABI calls"}
        else:  # real-valued inputs: fp32 rows in, final activations out
            e2e = e2e_fp32

    # ---- CPU oracle baseline (rank 0, N = 1 only), bounded sample
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        import oracle
        cores = os.cpu_count() or 1
        rows, T = oracle_sample_time(oracle, net, Yh, cores, args.cpu_seconds)
        cpu = {"value": rows * nnz / T, "unit": UNIT, "cores": cores, "kind": "oracle",
               "sample": f"{rows} of {B_local} rows, plain Eq. 1 oracle over all {net.L} layers ({T:.1f} s)",
               "cpu": cpu_info()}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": max(args.warmup, 3), "ms_per_step": ms, "higher_is_better": True, "scaling": args.scaling,
            "vs_baseline": None, "dtype": "f32", "data": "synthetic (seeded SDGC-like RadiX W, MNIST-like binary Y0)",
            "config": {"workload": f"{args.config}: {c['desc']}", "neurons": c["N"], "layers": c["L"],
                       "batch_per_rank": B_local, "global_batch": B_global, "connections": nnz, "w_mode": args.mode,
                       "t": t, "s": s, "n": snic["n"], "eta": 0.03, "eps": 0.03, "kernel": args.kernel,
                       "pre_fused": args.pre_fused,
                       "network_abi": "compact circulant" if isinstance(net, sdgc.CirculantNetwork) else "CSC",
                       "l2": "inputs larger than L2 (no flush)", "parallelism": f"dp{world} (row shards)"},
            "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "e2e_fp32_io": e2e_fp32, "clocks": clk,
            "gpu_launches": int(launches_per_step * args.steps),
            "uncompressed": unc, "phases_ms": phases,
            "dynamics": {k: st[k] for k in ("live_at_t", "n_centroids", "n_sampled", "residual_at_t",
                                            "residual_final", "n_categories")},
            "paper_context": "SNICIT 4096-480 on 1x RTX A6000, B=60000: 44.17 ms = 8.55e13 edges/s (Table 3, P:1377)",
        }
        print(json.dumps(line), flush=True)
    g.close()
    if distributed:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    return run_snicit(args)


if __name__ == "__main__":
    sys.exit(main())
