#!/usr/bin/env python
"""SNICIT hot-path benchmark: SDGC inference edges/s on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3] [--impl snicit|reference]

A step = one whole SNICIT inference (all SURVEY 8(a) rows: pre-convergence layers, conversion,
post-convergence layers, recovery, category set) over one batch.  The N = 1 workload is config C3
(SDGC 16384 neurons x 1920 layers, batch 60,000, t = 30, s = 32, n = 16, eta = eps = 0.03: the config
BASELINE.json quotes the metric "at 1/2/4/8 B200" on), synthetic inputs.

N > 1: one rank per GPU over NCCL.  `--gpus N` without a torchrun environment re-launches itself under
torch.distributed.run (127.0.0.1).  Default **strong** scaling: the one 60,000-row batch is
sharded in contiguous row blocks (B/G rows per rank, global ids by row_offset), weights replicated,
clustering per shard; the only collective is one all_gather of the per-rank category buffers, exported
on the device (snicit_categories_device, no host round trip).  `--scaling weak`: every rank its own batch.

value: device-resident inputs (Y0 already in HBM), CUDA events around exactly K steps on the stream the
library launches on, barrier + synchronize on both sides, max over ranks.  Inputs (3.9 GB at C3) exceed
L2 (126 MB): no flush needed.  e2e: the same metric through snicit_infer with pinned HOST
fp32 rows (H2D inside the call, streamed under the pre phase) and the category set read back to the host
(D2H); e2e_packed: the same through snicit_infer_packed (binary inputs as a bitmap).

Extra keys (N = 1): `residue` -- the method's conversion / residue kernels in a residue-heavy regime
(C2, t = 10) with their rooflines; `general_csc` -- the general (non-circulant) CSC path (C2 "perm"
weights) with the ELL layer kernel's HBM roofline.

--impl reference: the CPU oracle (plain Eq. 1, oracle/) timed on the host cores on a bounded row sample of
the same workload (rank 0 only; other ranks exit 0).
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


def parse(argv=None):
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=5)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", choices=["snicit", "reference"], default="snicit")
    p.add_argument("--config", default="C3", choices=["C1", "C2", "C3", "C4", "C5"])
    p.add_argument("--mode", default="radix", choices=["radix", "perm", "random"])
    p.add_argument("--t", type=int, default=None)
    p.add_argument("--s", type=int, default=None)
    p.add_argument("--kernel", default="auto", choices=["auto", "ell", "circ"])
    p.add_argument("--load", default="auto", choices=["auto", "csc", "compact"],
                   help="network ABI: explicit CSC (snicit_load_network) or compact circulant form; auto = "
                        "compact for radix nets with N >= 16384 (C3/C4 CSC is 8-32 GB)")
    p.add_argument("--scaling", default="strong", choices=["weak", "strong"])
    p.add_argument("--batch", type=int, default=None, help="override rows (strong: global, weak: per rank)")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-uncompressed", action="store_true")
    p.add_argument("--no-residue", action="store_true", help="skip the residue-regime study (C2, t = 10)")
    p.add_argument("--no-general", action="store_true", help="skip the general-CSC study (C2 perm)")
    p.add_argument("--residue-t", type=int, default=10)
    p.add_argument("--pre-fused", type=int, default=1, choices=[0, 1, 2, 3, 4, 5, 6, 7],
                   help="options.pre_fused: 1 = row-resident pre phase (default), 2 = without the constant-row "
                        "shortcut, 6 = without the range prediction (R30), 4 = rows split over a thread-block "
                        "cluster (N >= 16384), 0 = one launch per layer")
    p.add_argument("--no-variants", action="store_true", help="skip the pre_fused = 2 / 0 roofline variants")
    p.add_argument("--cpu-seconds", type=float, default=15.0, help="target CPU work of the oracle sample")
    p.add_argument("--quick", action="store_true", help="value only (no e2e/uncompressed/variants/studies)")
    p.add_argument("--dyn-log", default=os.path.join(ROOT, "gpurun_out", "bench_dynamics_{config}_rank{rank}.jsonl"),
                   help="per-layer dynamics JSONL of one inference per rank (SURVEY 5); '' = off")
    a = p.parse_args(argv)
    if a.quick:
        a.no_e2e = a.no_cpu_baseline = a.no_uncompressed = a.no_residue = a.no_general = a.no_variants = True
    return a


def config_params(args, config=None, t=None):
    config = config or args.config
    c = dict(sdgc.CONFIGS[config])
    if config == "C5":
        snic = dict(t=sdgc.medium_t(c["L"]), s=128, n=0)
    else:
        snic = dict(t=30, s=32, n=16)
    if t is not None:
        snic["t"] = t
    elif args.t is not None:
        snic["t"] = args.t
    if args.s is not None:
        snic["s"] = args.s
    if args.batch is not None and config == args.config:
        c["B"] = args.batch
    return c, snic


def use_compact(config, mode, load, c):
    if config == "C5" or mode != "radix":
        return False
    return load == "compact" or (load == "auto" and c["N"] >= 16384)


def make_network(config, mode, load, c):
    if config == "C5":
        return sdgc.gen_medium_network(c["N"], c["L"])
    if use_compact(config, mode, load, c):
        return sdgc.gen_circulant(c["N"], c["L"])
    return sdgc.gen_network(c["N"], c["L"], mode)


def oracle_layers(oracle, net, Y, nthreads=0):
    if isinstance(net, sdgc.CirculantNetwork):
        return oracle.layers_circulant_f32(net, Y, nthreads=nthreads)
    return oracle.layers_f32(net, Y, nthreads=nthreads)


def make_inputs(config, c, B, row0):
    if config == "C5":
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
                                          "--format=csv,noheader,nounits", "-lms", "20"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.th = threading.Thread(target=self._read, daemon=True)
            self.th.start()
            t0 = time.time()  # the sampler is producing lines before the timed region starts
            while not self.lines and time.time() - t0 < 10.0 and self.proc.poll() is None:
                time.sleep(0.02)
        except (OSError, FileNotFoundError):
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def mark(self):
        """Index of the next sample: samples from here on were taken during the timed region."""
        self.t_mark = len(self.lines)

    def stop(self):
        if self.proc is None:
            return None
        time.sleep(0.06)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, mx, reasons, pw = [], 0, set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        # samples of the timed region (plus the one straddling its end); at least the last one taken
        lines = self.lines[max(0, min(getattr(self, "t_mark", 0), len(self.lines) - 1)):]
        for ln in lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 8:
                continue
            try:
                sm.append(float(parts[0]))
                mx = max(mx, float(parts[1]))
                pw.append(float(parts[2]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return None
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": len(sm),
                "power_w_max": max(pw) if pw else None}


def gen_kernel_info(net):
    """(G, wavefronts per tap) of the general-CSC kernel for this network (kernels_gen.cu, DESIGN.md section
    7): G = outputs per warp instruction (0: the previous ELL kernels; SNICIT_GEN=0 forces those), and the
    load-time schedule's mean shared-memory wavefronts per quarter-warp tap over the first layers."""
    if os.environ.get("SNICIT_GEN", "1") == "0":
        return 0, None
    from paper_conf_icpp_jiangh0h23_b200.api import gen_schedule
    N = net.N
    costs, G = [], 0
    for l in range(min(3, net.L)):
        p = net.ptr[l * (N + 1):(l + 1) * (N + 1)]
        lens = np.diff(p)
        if lens.min() != lens.max():
            break
        cols = net.idx[p[0]:p[-1]].reshape(N, -1)
        G, cst = gen_schedule(cols)
        costs.append(cst)
    return G, (float(np.mean(costs)) if costs else None)


def gen_kernel_label(G):
    if G:
        return (f"layer_gen_kernel (general CSC, a1: row-interleaved tile of {128 // G} rows, "
                f"{G} outputs x 4 rows per lane group per warp instruction)")
    return "layer_ell_kernel (general CSC, a1)"


def committed_traffic(tag: str):
    """Mean DRAM bytes per launch of the dominant kernel from the latest committed ncu capture of this
    configuration (profiles/rNN_traffic_<tag>.json, written by scripts/traffic.py), or (None, None)."""
    import glob
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", f"r*_traffic_{tag}.json")))
    if not files:
        return None, None
    d = json.load(open(files[-1]))
    return float(d["mean_dram_bytes_per_launch"]), f"{os.path.basename(files[-1])} ({d['launches']} launches)"


# FP32 FMA pipe of a B200: 148 SMs x 128 FMA lanes/clk x 2 flop x 1965 MHz (B200_PROFILING.md: 148 SMs,
# clocks.max.sm 1965 MHz; 128 FP32 lanes per SM: scripts/ubench_ffma.cu measured 127.9 FMA/clk/SM,
# profiles/r02_ubench_ffma.txt)
FMA_PEAK_TFLOPS = 148 * 128 * 2 * 1965e6 / 1e12
FMA_PEAK_SRC = ("derived: 148 SMs x 128 FP32 FMA/clk x 2 flop x 1965 MHz = 74.45 TFLOP/s (DESIGN.md §7; "
                "scripts/ubench_ffma.cu measured 127.9 FMA/clk/SM, profiles/r02_ubench_ffma.txt)")


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


def oracle_sample_time(oracle, net, Y, cores, seconds, probe_only=False, max_rows=None):
    """Rows of Y the oracle processes in ~`seconds` on all host cores, and the measured time for them.
    Probe sizes double (from one row per core) until a probe takes >= seconds / 2: small probes are
    dominated by per-call and thread start-up cost, which would under-size the sample."""
    cap = len(Y) if max_rows is None else max_rows
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


def workload_config(args, c, snic, net, extra=None):
    d = {"workload": f"{args.config}: {c['desc']}", "neurons": c["N"], "layers": c["L"], "batch": c["B"],
         "connections": int(net.nnz), "w_mode": args.mode, "t": snic["t"], "s": snic["s"], "n": snic["n"],
         "eta": 0.03, "eps": 0.03}
    if extra:
        d.update(extra)
    return d


# ------------------------------------------------------------------ reference arm (CPU oracle)
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle

    c, snic = config_params(args)
    net = make_network(args.config, args.mode, args.load, c)
    nnz = net.nnz
    cores = os.cpu_count() or 1
    # size the per-step sample to ~cpu_seconds / steps of the oracle on all cores
    probe = make_inputs(args.config, c, min(c["B"], 64 * cores), 0)
    rows, _ = oracle_sample_time(oracle, net, probe, cores, args.cpu_seconds / max(args.steps, 1), probe_only=True,
                                 max_rows=c["B"])
    Y = make_inputs(args.config, c, rows, 0)
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
        "config": workload_config(args, c, snic, net),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample,
                         "cpu": cpu_info()},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ helpers of the SNICIT arm
def load_handle(net, dev_index):
    from paper_conf_icpp_jiangh0h23_b200 import SnicitNetwork
    if isinstance(net, sdgc.CirculantNetwork):
        return SnicitNetwork.circulant(net.N, net.L, net.nu, net.w, net.bias, net.ymax, device=dev_index)
    return SnicitNetwork.from_network(net, device=dev_index)


def event_ms(stream, fn, k, sync_dev):
    """CUDA-event time of k calls of fn on `stream` (synchronize on both sides)."""
    import torch
    torch.cuda.synchronize(sync_dev)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(k):
        fn()
    e1.record(stream)
    torch.cuda.synchronize(sync_dev)
    return e0.elapsed_time(e1) / k


def residue_study(args, dev, stream, peak):
    """The method's own conversion / residue kernels where they carry work: C2 at a small threshold
    layer (t = 10: ~31 centroids and ~23k non-empty residue rows, profiles/r01_studies.md).  Rooflines of
    map_residual_kernel (Alg. 2 / Eq. 3-4) and the residue trajectory kernel (Eq. 5) from live CUDA-event
    kernel times and the library's work counters."""
    from paper_conf_icpp_jiangh0h23_b200 import default_options
    cfg = "C2"
    c, snic = config_params(args, cfg, t=args.residue_t)
    net = make_network(cfg, "radix", "csc", c)
    Yh = make_inputs(cfg, c, c["B"], 0)
    g = load_handle(net, dev.index)
    g.set_stream(stream)
    import torch
    y0 = torch.from_numpy(Yh).to(dev)
    y_out = torch.empty_like(y0)
    t, s = snic["t"], snic["s"]
    opt = default_options(n_segments=snic["n"])

    def step():
        g.infer(y0, t=t, s=s, options=opt, y_out=y_out)
    step()
    ms = event_ms(stream, step, max(1, min(args.steps, 3)), dev)
    opt_t = default_options(n_segments=snic["n"], timing=2)
    g.infer(y0, t=t, s=s, options=opt_t, y_out=y_out)
    st = g.stats()
    N = c["N"]
    out = {"workload": f"C2 ({c['desc']}), t = {t}", "ms_per_step": ms, "value": c["B"] * net.nnz / (ms * 1e-3),
           "unit": UNIT, "phases_ms": {k: st[k] for k in ("t_pre_ms", "t_convert_ms", "t_post_ms", "t_recover_ms")},
           "dynamics": {k: st[k] for k in ("live_at_t", "n_centroids", "residual_at_t", "residual_final",
                                            "res_nnz_at_t", "res_full_rl", "res_sparse_rl", "res_sparse_out",
                                            "res_scalar_rl") if k in st}}
    kms = st.get("t_map_ms", -1.0)
    if kms and kms > 0:
        # map_residual (Alg. 2): the L0 distance of every mapped row to every centroid is map_rows x C x N
        # element comparisons.  Round 2 (r02c) compares each centroid element read from shared memory with 2-4 rows
        # (map_dist_kernel), so the bound is the ALU issue of a comparison -- a compare and an add per
        # element, 2 lane-ops: 148 SMs x 128 lanes x 1.965 GHz / 2 comparisons/s; `smem_equiv` keeps the
        # round-2 reading (one 4-byte shared read per comparison against 148 x 128 B/clk x 1.965 GHz).  HBM
        # moves 4 N per row read + 4 N per residue written (fraction reported alongside)
        comps = float(st.get("map_rows", 0)) * st["n_centroids"] * N
        cmp_peak = 148 * 128 * 1.965e9 / 2.0 / 1e12  # Tcomparisons/s
        ach_c = comps / (kms * 1e-3) / 1e12
        smem_peak = 148 * 128 * 1.965e9 / 1e9  # GB/s
        ach_s = 4.0 * comps / (kms * 1e-3) / 1e9
        by = 4.0 * N * (st["live_at_t"] + st["residual_at_t"])
        ach = by / (kms * 1e-3) / 1e9
        out["map_residual_kernel"] = {"bound": "alu", "achieved": ach_c, "peak": cmp_peak, "unit": "Tcomparisons/s",
                                      "frac": ach_c / cmp_peak, "ms": kms, "comparisons": comps,
                                      "peak_source": "derived: 148 SMs x 128 lanes x 1965 MHz / 2 lane-ops per comparison",
                                      "smem_equiv": {"achieved_gbs": ach_s, "peak_gbs": smem_peak, "frac": ach_s / smem_peak},
                                      "hbm": {"algorithmic_bytes": by, "achieved_gbs": ach, "frac": ach / peak}}
    rms = st.get("t_residual_ms", -1.0)
    if rms and rms > 0:
        # residue trajectories: 2 flop per evaluated tap (32 taps per evaluated output)
        outs = float(st.get("res_full_rl", 0)) * N + float(st.get("res_sparse_out", 0))
        flops = 2.0 * 32 * outs
        ach = flops / (rms * 1e-3) / 1e12
        out["residual_kernel"] = {"bound": "alu", "achieved": ach, "peak": FMA_PEAK_TFLOPS, "unit": "TFLOP/s",
                                  "frac": ach / FMA_PEAK_TFLOPS, "ms": rms, "algorithmic_flops": flops,
                                  "evaluated_outputs": outs, "peak_source": FMA_PEAK_SRC}
    # the same study with the dense-row residue form only (the paper's load-reduced SpMM)
    if "res_sparse_rl" in st:
        opt_d = default_options(n_segments=snic["n"], res_sparse=0)

        def step_d():
            g.infer(y0, t=t, s=s, options=opt_d, y_out=y_out)
        step_d()
        out["dense_residue_ms_per_step"] = event_ms(stream, step_d, max(1, min(args.steps, 3)), dev)
    g.close()
    del y0, y_out
    return out


def general_study(args, dev, stream, peak):
    """General (non-circulant) CSC path: C2 with "perm" weights (RadiX columns under a seeded output
    permutation per layer: 32 in / 32 out per neuron, not shift-invariant -> the ELL gather kernel).
    SURVEY 8(d): reported next to radix so structure-exploiting kernels cannot hide general-CSC speed."""
    from paper_conf_icpp_jiangh0h23_b200 import default_options
    cfg = "C2"
    c, snic = config_params(args, cfg, t=30)
    net = make_network(cfg, "perm", "csc", c)
    Yh = make_inputs(cfg, c, c["B"], 0)
    g = load_handle(net, dev.index)
    g.set_stream(stream)
    import torch
    y0 = torch.from_numpy(Yh).to(dev)
    y_out = torch.empty_like(y0)
    t, s = snic["t"], snic["s"]
    opt = default_options(n_segments=snic["n"])

    def step():
        g.infer(y0, t=t, s=s, options=opt, y_out=y_out)
    step()
    ms = event_ms(stream, step, max(1, min(args.steps, 3)), dev)
    g.infer(y0, t=t, s=s, options=default_options(n_segments=snic["n"], timing=2), y_out=y_out)
    pr = g.layer_profile()
    st = g.stats()
    kms, kb = float(pr["ms"].sum()), float(pr["bytes"].sum())
    ach = kb / (kms * 1e-3) / 1e9
    rows = float(pr["rows"].sum())
    # shared-memory gather ceiling: every fma needs its 4-byte input delivered from shared
    # memory to its lane; the L1 / shared data pipe delivers 128 B/clk/SM (148 SMs x 1.965 GHz)
    gather_peak = 148 * 128 * 1.965e9 / 4.0
    edge_rows = 32.0 * c["N"] * rows
    G, cost = gen_kernel_info(net)
    out = {"workload": f"C2 perm ({c['desc']}), t = {t}", "ms_per_step": ms, "value": c["B"] * net.nnz / (ms * 1e-3),
           "unit": UNIT, "circ_layers": st["circ_layers"],
           "roofline": {"bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak,
                        "kernel": gen_kernel_label(G), "launches": int(len(pr["ms"])),
                        "avg_launch_ms": kms / max(len(pr["ms"]), 1), "algorithmic_bytes": kb,
                        "edge_rows_per_s": edge_rows / (kms * 1e-3),
                        "smem_gather_frac": edge_rows / (kms * 1e-3) / gather_peak,
                        "smem_peak_gbs": gather_peak * 4 / 1e9, "schedule_wavefronts_per_tap": cost,
                        "hbm_ceiling_at_smem_peak": gather_peak * 4 / 1e9 / 16.0 / peak},
           "phases_ms": {k: st[k] for k in ("t_pre_ms", "t_convert_ms", "t_post_ms", "t_recover_ms")}}
    traffic, src = committed_traffic("C2_perm")
    out["roofline"]["traffic"] = traffic
    out["roofline"]["traffic_source"] = src
    g.close()
    return out


# ------------------------------------------------------------------ SNICIT arm
def run_snicit(args):
    import torch
    import torch.distributed as dist

    from paper_conf_icpp_jiangh0h23_b200 import (KERNEL_AUTO, KERNEL_CIRC, KERNEL_ELL, allgather_categories,
                                                 allgather_categories_padded, default_options, shard_capacity,
                                                 shard_rows)

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
        cap = c["B"]
    else:
        a, b = shard_rows(c["B"], world, rank)
        B_local, row0, B_global = b - a, a, c["B"]
        cap = shard_capacity(c["B"], world)
    net = make_network(args.config, args.mode, args.load, c)
    gen_G = gen_kernel_info(net)[0] if isinstance(net, sdgc.Network) else 0
    nnz = net.nnz
    kern = {"auto": KERNEL_AUTO, "ell": KERNEL_ELL, "circ": KERNEL_CIRC}[args.kernel]
    Yh = make_inputs(args.config, c, B_local, row0)
    g = load_handle(net, dev.index)
    stream = torch.cuda.Stream(device=dev)
    g.set_stream(stream)
    y0 = torch.from_numpy(Yh).to(dev)
    y_out = torch.empty_like(y0)
    cat_buf = torch.empty(1 + cap, dtype=torch.int64, device=dev)
    opt = default_options(kernel=kern, n_segments=snic["n"], pre_fused=args.pre_fused)
    t, s = snic["t"], snic["s"]
    gathered = [None]

    def step():
        g.infer(y0, t=t, s=s, options=opt, y_out=y_out, row_offset=row0)
        g.categories_device(cat_buf)  # [count, ids...] on the device, queued on the library's stream
        if distributed:
            with torch.cuda.stream(stream):
                gathered[0] = allgather_categories_padded(cat_buf if backend == "nccl" else cat_buf.cpu())

    def timed(fn, k):
        if distributed:
            dist.barrier()
        ms = event_ms(stream, fn, k, dev)
        if distributed:
            dist.barrier()
            tt = torch.tensor([ms], device=coll_dev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            ms = float(tt.item())
        return ms

    clocks = ClockSampler(dev.index)
    if rank == 0:
        clocks.start()  # running (and under load through the warm-up) before the timed region
    for _ in range(max(args.warmup, 3)):
        step()
    if rank == 0:
        clocks.mark()
    ms = timed(step, args.steps)
    clk = clocks.stop() if rank == 0 else None
    st0 = g.stats()
    launches_per_step = st0["kernel_launches"]
    value = B_global * nnz / (ms * 1e-3)
    n_cat_global = None
    if distributed:
        counts = gathered[0][:, 0].tolist()
        n_cat_global = int(sum(counts))
    else:
        n_cat_global = int(cat_buf[0].item())

    # ---- per-rank phase times (one extra inference with phase events)
    g.infer(y0, t=t, s=s, options=default_options(kernel=kern, n_segments=snic["n"], pre_fused=args.pre_fused,
                                                  timing=1), y_out=y_out, row_offset=row0)
    st1 = g.stats()
    dyn_path = None
    if args.dyn_log:
        dyn_path = args.dyn_log.format(config=args.config, rank=rank)
        os.makedirs(os.path.dirname(dyn_path) or ".", exist_ok=True)
        g.write_dynamics_jsonl(dyn_path, {"config": args.config, "rank": rank, "row_offset": row0})
    mine = {"rank": rank, "rows": B_local, "row_offset": row0,
            **{k: st1[k] for k in ("t_pre_ms", "t_convert_ms", "t_post_ms", "t_recover_ms", "t_total_ms",
                                   "live_at_t", "n_centroids", "residual_at_t", "n_categories")}}
    per_rank = [mine]
    if distributed:
        per_rank = [None] * world
        dist.all_gather_object(per_rank, mine)

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

    peak, peak_src = measured_peaks()
    roof = None
    phases = {k: st1[k] for k in ("t_pre_ms", "t_convert_ms", "t_post_ms", "t_recover_ms", "t_total_ms")}
    if rank == 0 or not distributed:
        st, pm, pb = profile_pre(args.pre_fused)
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
                            "layer_circ_col_kernel (strided)") if st_["circ_layers"] else gen_kernel_label(gen_G),
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
                                      "frac": round(b_ / (ms_ * 1e-3) / 1e9 / peak, 4)}
                                  for k, (n, ms_, b_) in by.items()}
            return r

        def alu_roof(pm_, pb_, st_):
            """FP32 FMA-pipe roofline of the row-resident kernel: algorithmic flops = 2 x 32 x N (Eq. 1) per
            evaluated row-layer -- by fma chains, or by the popcount table of R32 (the layer is evaluated
            exactly, its Eq. 1 work counted however it is done); row-layers skipped by the exact shortcuts
            (constant rows R26, range prediction R30, bounds R31 / R34) are not evaluated and not counted."""
            kms = float(pm_.sum())
            popc_rl = float(st_.get("pre_popc_rows", 0))
            flops = 2.0 * 32 * c["N"] * (float(st_["pre_full_rows"]) + popc_rl)
            achieved = flops / (kms * 1e-3) / 1e12
            hbm_gbs = float(pb_.sum()) / (kms * 1e-3) / 1e9
            traffic, traffic_src = committed_traffic(tag + "_fused") if tag else (None, None)
            return {"bound": "alu", "achieved": achieved, "peak": FMA_PEAK_TFLOPS, "unit": "TFLOP/s",
                    "frac": achieved / FMA_PEAK_TFLOPS, "traffic": traffic,
                    "traffic_unit": "bytes per launch (ncu dram read + write)", "traffic_source": traffic_src,
                    "kernel": ("pre_cluster_kernel (row-resident a1, a row split over a cluster of N/8192 CTAs, "
                               "DSMEM exchange)") if st_["pre_fused"] == 2 else
                              "pre_fused_kernel (row-resident a1: layers 0..t-1 of a row in shared memory)",
                    "peak_source": FMA_PEAK_SRC, "launches": int(len(pm_)), "avg_launch_ms": kms,
                    "algorithmic_flops": flops, "full_row_layers": int(st_["pre_full_rows"]),
                    "popcount_row_layers": int(popc_rl),
                    "const_rows": int(st_["pre_const_rows"]),
                    "hbm": {"algorithmic_bytes": float(pb_.sum()), "achieved_gbs": hbm_gbs, "frac": hbm_gbs / peak,
                            "peak": peak, "peak_source": peak_src}}

        if len(pm):
            roof = alu_roof(pm, pb, st) if st["pre_fused"] else hbm_roof(pm, pb, st)
            # the timed step of a rank processes B_local rows; roofline launches are this rank's too
            roof["share_of_step"] = float(pm.sum() / ms) if ms > 0 else None
            if st["pre_fused"] and ms > 0:
                step_flops = roof["algorithmic_flops"]
                step_bytes = roof["hbm"]["algorithmic_bytes"] + 4.0 * c["N"] * st["live_at_t"]
                roof["whole_step"] = {"alu_frac": step_flops / (ms * 1e-3) / 1e12 / FMA_PEAK_TFLOPS,
                                      "hbm_frac": step_bytes / (ms * 1e-3) / 1e9 / peak,
                                      "algorithmic_flops": step_flops, "algorithmic_bytes": step_bytes}
            if st["pre_fused"] and not args.no_variants:
                st2, pm2, pb2 = profile_pre(2)
                if st2["pre_fused"] and len(pm2):
                    r2 = alu_roof(pm2, pb2, st2)
                    roof["no_const_skip"] = {k: r2[k] for k in ("achieved", "frac", "avg_launch_ms",
                                                                "full_row_layers")}
                st6, pm6, pb6 = profile_pre(6)
                if st6["pre_fused"] and len(pm6):
                    r6 = alu_roof(pm6, pb6, st6)
                    roof["no_range_pred"] = {k: r6[k] for k in ("achieved", "frac", "avg_launch_ms",
                                                                "full_row_layers")}
                st0_, pm0, pb0 = profile_pre(0)
                if len(pm0):
                    r0 = hbm_roof(pm0, pb0, st0_)
                    roof["per_layer_kernels"] = {k: r0[k] for k in ("bound", "achieved", "peak", "unit", "frac",
                                                                    "traffic", "traffic_source", "launches",
                                                                    "avg_launch_ms", "by_stride") if k in r0}
                    roof["per_layer_kernels"]["ms_total"] = float(pm0.sum())

    # ---- dynamic threshold layer (options.dyn_t, DESIGN R28): t chosen from the first s rows, at most t
    dyn = None
    if not args.no_uncompressed:
        opt_d = default_options(kernel=kern, n_segments=snic["n"], pre_fused=args.pre_fused, dyn_t=1)

        def step_dyn():
            g.infer(y0, t=t, s=s, options=opt_d, y_out=y_out, row_offset=row0)
            g.categories_device(cat_buf)
        step_dyn()
        ms_d = timed(step_dyn, max(1, min(args.steps, 3)))
        dyn = {"t": int(g.stats()["threshold_layer"]), "t_max": t, "ms_per_step": ms_d,
               "value": B_global * nnz / (ms_d * 1e-3), "unit": UNIT}

    # ---- uncompressed GPU baseline (t >= L, same kernels)
    unc = None
    if not args.no_uncompressed:
        def step_unc():
            g.infer(y0, t=net.L, s=s, options=opt, y_out=y_out, row_offset=row0)
            g.categories_device(cat_buf)
            if distributed:
                with torch.cuda.stream(stream):
                    allgather_categories_padded(cat_buf if backend == "nccl" else cat_buf.cpu())
        step_unc()
        ms_u = timed(step_unc, max(1, min(args.steps, 3)))
        unc = {"value": B_global * nnz / (ms_u * 1e-3), "unit": UNIT, "ms_per_step": ms_u,
               "speedup_snicit": ms_u / ms, "pre_fused": args.pre_fused}
        if args.pre_fused and not args.no_variants:  # plain layer-by-layer launches (no row residency)
            opt0 = default_options(kernel=kern, n_segments=snic["n"], pre_fused=0)

            def step_unc0():
                g.infer(y0, t=net.L, s=s, options=opt0, y_out=y_out, row_offset=row0)
                g.categories_device(cat_buf)
                if distributed:
                    with torch.cuda.stream(stream):
                        allgather_categories_padded(cat_buf if backend == "nccl" else cat_buf.cpu())
            step_unc0()
            ms_u0 = timed(step_unc0, max(1, min(args.steps, 3)))
            unc["per_layer_kernels"] = {"value": B_global * nnz / (ms_u0 * 1e-3), "ms_per_step": ms_u0}

    # ---- e2e through the C ABI with host (pinned) buffers: snicit_infer with fp32 Y0 from
    # the host (H2D inside the call, streamed under the pre phase) and the category set read back (D2H),
    # all-gathered across ranks.  Also: snicit_infer_packed (binary inputs as a bitmap).
    e2e = e2e_packed = None
    if not args.no_e2e:
        from paper_conf_icpp_jiangh0h23_b200 import pack_rows
        binary = bool(np.all((Yh == 0) | (Yh == 1)))  # SDGC inputs; config 5's are real-valued
        yh_pin = torch.from_numpy(Yh).pin_memory()
        bits_pin = torch.from_numpy(pack_rows(Yh).view(np.int32)).pin_memory() if binary else None

        def gather_host(cats):
            if distributed:
                with torch.cuda.stream(stream):
                    allgather_categories(torch.from_numpy(cats).to(coll_dev))

        def step_fp32():
            g.infer(yh_pin.numpy(), t=t, s=s, options=opt, row_offset=row0)  # host y0: returns when consumed
            cats = g.categories()
            gather_host(cats)
            return cats

        def step_packed():
            g.infer_packed(bits_pin.numpy(), t=t, s=s, options=opt, row_offset=row0)
            cats = g.categories()
            gather_host(cats)
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
        e2e = {"value": B_global * nnz / (ms_f * 1e-3), "unit": UNIT, "ms_per_step": ms_f,
               "h2d_bytes_per_step": int(Yh.nbytes) * world, "d2h_bytes_per_step": (4 + 8 * len(cats)) * world,
               "api": "snicit_infer (fp32 Y0 from pinned host memory, streamed H2D under the pre phase) + "
                      "snicit_categories (D2H)",
               "timer": "host wall clock around K synchronous C-ABI calls, max over ranks"}
        if binary:
            ms_e, cats = wall(step_packed)
            e2e_packed = {"value": B_global * nnz / (ms_e * 1e-3), "unit": UNIT, "ms_per_step": ms_e,
                          "h2d_bytes_per_step": int(bits_pin.numel() * 4) * world,
                          "d2h_bytes_per_step": (4 + 8 * len(cats)) * world,
                          "api": "snicit_infer_packed (Y0 as packed binary bitmap) + snicit_categories",
                          "timer": "host wall clock around K synchronous C-ABI calls, max over ranks"}

    # ---- studies of the method's own kernels (rank 0, N = 1)
    residue = general = None
    if rank == 0 and not distributed:
        if not args.no_residue and args.config != "C5":
            residue = residue_study(args, dev, stream, peak)
        if not args.no_general and args.config != "C5":
            general = general_study(args, dev, stream, peak)

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
            "config": workload_config(args, c, snic, net, {
                "batch_per_rank": B_local, "global_batch": B_global, "kernel": args.kernel,
                "pre_fused": args.pre_fused,
                "network_abi": "compact circulant" if isinstance(net, sdgc.CirculantNetwork) else "CSC",
                "l2": "inputs larger than L2 (no flush)",
                "parallelism": f"dp{world} (row shards, {args.scaling} scaling)"}),
            "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "e2e_packed": e2e_packed, "clocks": clk,
            "gpu_launches": int(launches_per_step * args.steps + (2 * args.steps if distributed else args.steps)),
            "uncompressed": unc, "dynamic_t": dyn, "phases_ms": phases, "per_rank": per_rank,
            "categories": n_cat_global,
            "dynamics": {k: st0[k] for k in ("live_at_t", "n_centroids", "n_sampled", "residual_at_t",
                                             "residual_final", "n_categories")},
            "residue": residue, "general_csc": general, "dynamics_log": dyn_path,
            "paper_context": "SNICIT 16384-1920 on 1x RTX A6000, B=60000: 179.37 ms = 3.37e14 edges/s "
                             "(Table 3, P:1383)",
        }
        print(json.dumps(line), flush=True)
    g.close()
    if distributed:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def spawn(args, argv):
    """`--gpus N` outside a torchrun environment: re-launch this script with N ranks (one per GPU)."""
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")        # keep NCCL's communicator log (init, NVLS) on stderr
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    import socket
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + argv
    return subprocess.call(cmd, env=env)


def main(argv=None):
    argv = sys.argv[1:] if argv is None else argv
    args = parse(argv)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return spawn(args, argv)
    if args.impl == "reference":
        return run_reference(args)
    return run_snicit(args)


if __name__ == "__main__":
    sys.exit(main())
