#!/usr/bin/env python
"""bench.py -- WY-based SBR on B200: the BASELINE.json headline metric.

Metric (BASELINE.json): SBR seconds and effective TFLOP/s = (4/3) n^3 / seconds at
n=32768, b=32 (config 4: random symmetric, nb=1024, FP16-in/FP32-acc mode), as a
fraction of B200 tensor peak.  A "step" is one full sbr_reduce (all of SURVEY
§8(a): panels, lazy updates, W merges, passes, trailing SYR2Ks, band extraction)
over one synthetic n x n input resident in HBM.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

One process per GPU (torchrun for N>1; a plain `--gpus N` re-launches itself under
torch.distributed.run).  N>1 reduces ONE matrix across the ranks with sbr_reduce_dist (strong
scaling, "scaling": "strong"): 1D block-cyclic nb-column blocks, the owner of each block
factors its panels and NCCL-broadcasts W_t, every rank streams the pass tiles and applies the
SYR2K on its own columns; every rank times its own steps and the max
over ranks is reported.
``--impl reference`` times the CPU oracle (this tier has no reference implementation; the
oracle is the reference arm).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIG4 = {"n": 32768, "b": 32, "nb": 1024, "mode": "fp16", "kind": "random_symmetric"}
METRIC = "SBR seconds & effective TFLOPS ((4/3)n³) at n=32768,b=32 vs B200 tensor peak"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=5)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--n", type=int, default=CONFIG4["n"])
    p.add_argument("--b", type=int, default=CONFIG4["b"])
    p.add_argument("--nb", type=int, default=CONFIG4["nb"])
    p.add_argument("--mode", default=CONFIG4["mode"])
    p.add_argument("--input", default="uniform", choices=["uniform", "geo"],
                   help="uniform: random symmetric U[-1,1) (configs 1, 3, 4); geo: prescribed spectrum "
                        "SVD_Geo kappa=1e5 (configs 2, 5)")
    p.add_argument("--e2e-steps", type=int, default=2)
    p.add_argument("--form-q-steps", type=int, default=1,
                   help="also time sbr_form_q (Q = prod (I - W Y^T), 3xTF32) on the last step's output (0: skip)")
    p.add_argument("--profile-steps", type=int, default=2)
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--cpu-sample-s", type=float, default=15.0)
    p.add_argument("--lapack-n", type=int, default=16384,
                   help="n of the LAPACK ssytrd_sy2sb/dsytrd_sy2sb host baseline (0: skip)")
    return p.parse_args()


def eff_tflops(n: int, seconds: float) -> float:
    return (4.0 / 3.0) * n ** 3 / seconds / 1e12


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback"


class ClockSampler:
    """Samples SM clock and throttle reasons via NVML while the timed region runs."""

    def __init__(self, index: int):
        self.index = index
        self.samples = []
        self.reasons = set()
        self.sm_max = None
        self._stop = threading.Event()
        self._t = None

    def __enter__(self):
        try:
            import pynvml as nv

            nv.nvmlInit()
            self._nv = nv
            self._h = nv.nvmlDeviceGetHandleByIndex(self.index)
            self.sm_max = nv.nvmlDeviceGetMaxClockInfo(self._h, nv.NVML_CLOCK_SM)
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        except Exception as e:  # pragma: no cover
            self._err = str(e)
        return self

    def _run(self):
        nv = self._nv
        names = {
            "gpu_idle": getattr(nv, "nvmlClocksEventReasonGpuIdle", 0x1),
            "sw_power_cap": getattr(nv, "nvmlClocksEventReasonSwPowerCap", 0x4),
            "hw_slowdown": getattr(nv, "nvmlClocksEventReasonHwSlowdown", 0x8),
            "sw_thermal_slowdown": getattr(nv, "nvmlClocksEventReasonSwThermalSlowdown", 0x20),
            "hw_thermal_slowdown": getattr(nv, "nvmlClocksEventReasonHwThermalSlowdown", 0x40),
            "hw_power_brake_slowdown": getattr(nv, "nvmlClocksEventReasonHwPowerBrakeSlowdown", 0x80),
        }
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self._h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self._h)
                for k, bit in names.items():
                    if r & bit and k != "gpu_idle":
                        self.reasons.add(k)
            except Exception:
                pass
            self._stop.wait(0.1)

    def __exit__(self, *exc):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        med = statistics.median(self.samples) if self.samples else None
        return {"sm_mhz": med, "sm_max_mhz": self.sm_max, "reasons": sorted(self.reasons),
                "samples": len(self.samples)}


def cpu_oracle_sample(n: int, b: int, a_host, budget_s: float):
    """Time the CPU oracle (oracle.sbr.sbr_unblocked, fp64 numpy, as it stands) on a prefix of
    the same n x n reduction and extrapolate: setup (measured) + loop time scaled by the
    per-column cost (n - c - b) of the remaining columns."""
    import numpy as np

    from oracle import sbr as osbr

    ncol_total = max(0, n - b - 1)
    st = {}
    t0 = time.perf_counter()
    osbr.sbr_unblocked(a_host, b, want_q=False, max_cols=1, stats=st)
    t_first = time.perf_counter() - t0
    per_col = max(st["loop_seconds"], 1e-6)
    setup = max(t_first - st["loop_seconds"], 0.0)
    cols = int(max(1, min(ncol_total, (budget_s - setup) / per_col)))
    st = {}
    osbr.sbr_unblocked(a_host, b, want_q=False, max_cols=cols, stats=st)
    c = np.arange(ncol_total, dtype=np.float64)
    w = (n - c - b)
    frac = float(w[:cols].sum() / w.sum())
    t_full = setup + st["loop_seconds"] / frac
    cores = len(os.sched_getaffinity(0))
    try:
        from threadpoolctl import threadpool_info

        thr = max((i.get("num_threads", 1) for i in threadpool_info()), default=cores)
    except Exception:
        thr = cores
    return {
        "value": eff_tflops(n, t_full),
        "unit": "TFLOP/s",
        "cores": int(thr),
        "kind": "oracle",
        "sample": f"oracle.sbr.sbr_unblocked (fp64 numpy, as it stands) on the first {cols} of {ncol_total} "
                  f"columns of the same n={n} b={b} input: setup {setup:.1f} s + {st['loop_seconds']:.1f} s loop, "
                  f"extrapolated by per-column cost (n-c-b) to ~{t_full:.3g} s for the full reduction",
        "seconds_extrapolated": t_full,
    }


def lapack_sy2sb_baseline(n_lapack: int, b: int, n_target: int, seed: int):
    """LAPACK ssytrd_sy2sb / dsytrd_sy2sb (UPLO='L', kd=b) from scipy's bundled OpenBLAS on all
    host cores (north_star / BASELINE.md §4): the same reduction (entry-wise equal up to
    rounding) in fp32 and fp64, at n_lapack (bounded: finishes in seconds), reported
    as effective TFLOP/s ((4/3) n^3) and extrapolated by n^3 to n_target."""
    import ctypes
    import glob

    import numpy as np
    import scipy

    import workloads

    d = os.path.join(os.path.dirname(scipy.__file__), "..", "scipy.libs")
    cands = sorted(glob.glob(os.path.join(d, "libscipy_openblas*.so")))
    if not cands:
        return None
    lib = ctypes.CDLL(cands[0])
    a0 = workloads.random_symmetric(n_lapack, seed)
    out = {}
    for name, dtype, fn in (("ssytrd_sy2sb", np.float32, "scipy_ssytrd_sy2sb_"),
                            ("dsytrd_sy2sb", np.float64, "scipy_dsytrd_sy2sb_")):
        if not hasattr(lib, fn):
            continue
        f = getattr(lib, fn)
        n = n_lapack
        af = np.asfortranarray(a0.astype(dtype))
        ab = np.zeros((b + 1, n), dtype=dtype, order="F")
        tau = np.zeros(max(1, n - b), dtype=dtype)
        info = ctypes.c_int(0)
        uplo = ctypes.c_char(b"L")
        i32 = ctypes.c_int
        ptr = lambda x: x.ctypes.data_as(ctypes.c_void_p)  # noqa: E731
        wq = np.zeros(1, dtype=dtype)
        args = [ctypes.byref(uplo), ctypes.byref(i32(n)), ctypes.byref(i32(b)), ptr(af), ctypes.byref(i32(n)),
                ptr(ab), ctypes.byref(i32(b + 1)), ptr(tau)]
        f(*args, ptr(wq), ctypes.byref(i32(-1)), ctypes.byref(info), ctypes.c_size_t(1))
        work = np.zeros(max(1, int(wq[0])), dtype=dtype)
        t0 = time.perf_counter()
        f(*args, ptr(work), ctypes.byref(i32(work.size)), ctypes.byref(info), ctypes.c_size_t(1))
        dt = time.perf_counter() - t0
        out[name] = {"seconds": dt, "n": n, "tflops": eff_tflops(n, dt),
                     "extrapolated_seconds_at_n_target": dt * (n_target / n) ** 3, "info": info.value}
    try:
        from threadpoolctl import threadpool_info

        thr = max((i.get("num_threads", 1) for i in threadpool_info() if "openblas" in i.get("internal_api", "")),
                  default=len(os.sched_getaffinity(0)))
    except Exception:
        thr = len(os.sched_getaffinity(0))
    out["cores"] = int(thr)
    out["host_cpus"] = len(os.sched_getaffinity(0))
    out["note"] = (f"LAPACK (scipy OpenBLAS) dense->band, UPLO=L, kd={b}, on the same seeded generator at "
                   f"n={n_lapack} (bounded; n^3-extrapolated to n={n_target})")
    return out


def dist_setup():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        import torch.distributed as dist

        dist.init_process_group("nccl" if os.environ.get("SBR_BENCH_GLOO") is None else "gloo")
    return rank, world, local


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle, as it stands, on bounded samples of config 4.

    Each step runs oracle.sbr.sbr_unblocked on the same n x n input for one column (its
    setup plus one column of the plain unblocked reduction) and extrapolates the full
    reduction time by the per-column cost (n - c - b); value = (4/3) n^3 / that time."""
    if rank != 0:
        return
    import numpy as np

    import workloads
    from oracle import sbr as osbr

    n, b = args.n, args.b
    a_host = workloads.random_symmetric(n, workloads.config_seed(4))
    ncol_total = max(0, n - b - 1)
    w = (n - np.arange(ncol_total, dtype=np.float64) - b)
    # the oracle's setup (fp64 copy + symmetrisation of the n x n input) is timed once; every
    # step then times ONE column of the plain unblocked reduction on that input, and the full
    # reduction time is extrapolated by the per-column cost (n - c - b)
    st = {}
    t0 = time.perf_counter()
    osbr.sbr_unblocked(a_host, b, want_q=False, max_cols=1, stats=st)
    setup = time.perf_counter() - t0 - st["loop_seconds"]
    vals, last = [], None
    for i in range(args.warmup + args.steps):
        st = {}
        osbr.sbr_unblocked(a_host, b, want_q=False, max_cols=1, stats=st)
        t_full = setup + st["loop_seconds"] * float(w.sum() / w[0])
        if i >= args.warmup:
            vals.append(eff_tflops(n, t_full))
            last = (setup, st["loop_seconds"], t_full)
    v = statistics.median(vals)
    cores = len(os.sched_getaffinity(0))
    sample = (f"per step: oracle.sbr.sbr_unblocked (fp64 numpy, as it stands) on the n={n} b={b} input for 1 "
              f"of {ncol_total} columns ({last[1]:.2f} s; the oracle's setup, {last[0]:.1f} s, timed once), "
              f"extrapolated by per-column cost (n-c-b) to ~{last[2]:.3g} s for the full reduction")
    line = {
        "impl": "reference",
        "metric": METRIC, "value": v, "unit": "TFLOP/s", "n_gpus": args.gpus, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": (4.0 / 3.0) * n ** 3 / (v * 1e12) * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"config4: n={n} random symmetric, b={b}, nb={args.nb} (oracle is unblocked)",
                   "n": n, "b": b, "nb": args.nb, "parallelism": "cpu"},
        "cpu_baseline": {"value": v, "unit": "TFLOP/s", "cores": cores, "kind": "oracle", "sample": sample},
        "e2e": {"value": v, "unit": "TFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def respawn_distributed(args):
    """`python bench.py --gpus N` without a torchrun environment: re-launch under
    torch.distributed.run with N local ranks (127.0.0.1) and exit with its status."""
    import subprocess

    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", os.environ.get("SBR_BENCH_PORT", "29517"),
           os.path.abspath(__file__)] + sys.argv[1:]
    sys.exit(subprocess.call(cmd))


def main():
    args = parse()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        respawn_distributed(args)
    rank, world, local = dist_setup()
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    import numpy as np
    import torch

    torch.cuda.set_device(local)
    import __graft_entry__

    __graft_entry__.build()
    import paper_conf_ppopp_zhangsoyw23_b200 as sbr
    import workloads

    n, b, nb, mode = args.n, args.b, args.nb, args.mode
    cfg_name = {(32768, 32, 1024, "fp16"): "config4", (16384, 32, 1024, "3xtf32"): "config3",
                (4096, 32, 256, "fp16"): "config2", (65536, 64, 2048, "3xtf32"): "config5",
                (65536, 64, 2048, "3xtf32"): "config5-params"}.get((n, b, nb, mode), "custom")
    seed = workloads.config_seed({"config2": 2, "config3": 3, "config5": 5, "config5-params": 5}.get(cfg_name, 4))
    stream = torch.cuda.current_stream()
    if world > 1:
        # one matrix across the ranks (sbr_reduce_dist, strong scaling): NCCL communicator
        # from a unique id that rank 0 creates and torch.distributed carries
        uid = [sbr.get_unique_id() if rank == 0 else None]
        torch.distributed.broadcast_object_list(uid, src=0)
        h = sbr.Handle(local, stream, unique_id=uid[0], rank=rank, nranks=world)
    else:
        h = sbr.Handle(local, stream)
    if args.input == "uniform":
        pristine = h.generate_symmetric(seed, n)          # device twin of workloads.random_symmetric
        input_desc = f"random symmetric U[-1,1) (seed {seed})"
    else:   # prescribed spectrum, SVD_Geo kappa = 1e5: Haar Q (host) or randomised Hadamard Q (device)
        pristine, input_desc = workloads.prescribed_spectrum_device(n, "geo", 1e5, seed, a_device=f"cuda:{local}")
    if world > 1:   # 1D block-cyclic: this rank keeps only its nb-blocks of columns
        cols = torch.from_numpy(sbr.local_columns(n, nb, rank, world)).to(pristine.device)
        pristine = pristine.index_select(0, cols).contiguous()
        torch.cuda.empty_cache()
    a = torch.empty_like(pristine)
    ab = torch.empty((n, b + 1), dtype=torch.float32, device=a.device) if rank == 0 else None
    w = torch.zeros((a.shape[0], n), dtype=torch.float32, device=a.device) if world > 1 else \
        torch.empty((n - b, n), dtype=torch.float32, device=a.device)

    def run_step():
        if world > 1:
            h.reduce_dist(a, n, b, nb, mode=mode, ab=ab, w=w)
        else:
            h.reduce(a, b, nb, mode=mode, ab=ab, w=w)

    # warm-up (untimed)
    for _ in range(args.warmup):
        a.copy_(pristine)
        run_step()
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    # timed region: K steps, each bracketed by CUDA events on the launching stream; the
    # input is restored from the pristine copy between steps, outside the events.  No
    # per-kernel events here (they would serialise the programmatic dependent launches).
    launches0 = h.launch_count()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        for i in range(args.steps):
            a.copy_(pristine)
            evs[i][0].record(stream)
            run_step()
            evs[i][1].record(stream)
        torch.cuda.synchronize()
    launches = h.launch_count() - launches0
    step_ms = [e0.elapsed_time(e1) for e0, e1 in evs]
    total_ms = sum(step_ms)
    # profiled steps (right after the timed region, same stream): CUDA events around every
    # kernel class give the per-kernel durations behind `roofline` and `breakdown`
    h.reset_kernel_stats()
    h.set_kernel_timing(True)
    prof_ms = []
    for _ in range(args.profile_steps):
        a.copy_(pristine)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        run_step()
        e1.record(stream)
        torch.cuda.synchronize()
        prof_ms.append(e0.elapsed_time(e1))
    h.set_kernel_timing(False)
    if world > 1:
        t = torch.tensor([total_ms], device=a.device)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        torch.distributed.barrier()
        total_ms = float(t.item())
    ms_per_step = total_ms / args.steps
    value = eff_tflops(n, ms_per_step / 1e3)   # one n x n matrix per step, on all ranks together

    # per-kernel-class stats (events around every launch inside the timed region)
    classes = ["panel", "lazy", "wmerge", "pass", "syr2k", "other"]
    kst = {c: h.kernel_stats(c) for c in classes}
    dom = max(["pass", "syr2k", "panel", "lazy", "wmerge"], key=lambda c: kst[c]["ms"])
    peaks, src = load_peaks()
    st = kst[dom]
    nprof = max(1, args.profile_steps)
    avg_ms = st["ms"] / max(1, st["launches"])
    if dom == "syr2k":
        achieved = st["flops"] / max(1, st["launches"]) / (avg_ms / 1e3) / 1e12
        peak = peaks.get("bf16_tflops_sustained", peaks.get("bf16_tflops"))
        if mode == "3xtf32":   # tf32 dense peak = bf16 x the guide's nominal ratio 1.125 / 2.25
            peak *= 0.5
        roof = {"bound": "tensor", "achieved": achieved, "peak": peak, "unit": "TFLOP/s",
                "frac": achieved / peak, "traffic": None}
    else:
        achieved = st["bytes"] / max(1, st["launches"]) / (avg_ms / 1e3) / 1e9
        peak = peaks["hbm_gbs"]
        roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": None}
    # traffic: DRAM bytes per algorithmic byte of this kernel from the committed `ncu --set full`
    # capture (profiles/traffic.json), times this run's algorithmic bytes per launch
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            tr = json.load(f).get(f"{dom}:{mode}")   # captures are per kernel AND mode (fp16 / 3xtf32 kernels differ)
        if tr:
            roof["traffic"] = tr["dram_per_algorithmic_byte"] * st["bytes"] / max(1, st["launches"])
            roof["traffic_source"] = tr["source"]
    except Exception:
        pass
    roof.update({"kernel": dom, "peak_source": src, "launches_per_step": st["launches"] / nprof, "avg_ms": avg_ms,
                 "share_of_step": st["ms"] / sum(prof_ms) if prof_ms else None,
                 "measured_on": f"{nprof} profiled step(s) right after the timed region, CUDA events around every "
                                f"kernel class on the launching stream ({statistics.mean(prof_ms):.1f} ms/step with "
                                f"the events)"})
    breakdown = {c: {"ms_per_step": kst[c]["ms"] / nprof, "launches_per_step": kst[c]["launches"] / nprof}
                 for c in classes}

    # sbr_form_q on the profiled step's output: not part of the step, reported beside it
    formq = None
    if args.form_q_steps > 0 and world == 1 and n > b:
        q = torch.empty((n, n), dtype=torch.float32, device=a.device)
        fq_ms = []
        for _ in range(args.form_q_steps + 1):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            h.form_q(a, w, b, nb, q=q)
            e1.record(stream)
            torch.cuda.synchronize()
            fq_ms.append(e0.elapsed_time(e1))
        fq = statistics.median(fq_ms[1:])
        ncols = n - b
        alg = sum(4.0 * (n - c0 - b) ** 2 * min(nb, ncols - c0) for c0 in range(0, ncols, nb))
        formq = {"ms": fq, "algorithmic_tflops": alg / (fq / 1e3) / 1e12,
                 "tensor_tflops_3xtf32": 3 * alg / (fq / 1e3) / 1e12, "steps": args.form_q_steps,
                 "note": "Q = prod_J (I - W_J Y_J^T) by backward accumulation, 2 tcgen05 3xTF32 products per "
                         "block, algorithmic flops sum_J 4 M_J^2 k_J; first call (allocation) untimed"}
        del q

    # end-to-end through the public API with HOST buffers (H2D of A + D2H of the band per step)
    e2e = None
    if args.e2e_steps > 0 and world > 1:
        # every rank copies the pinned host input in, the ranks reduce it together, rank 0
        # reads the band back; wall clock with a barrier on both sides, max over ranks
        a_host = torch.empty(tuple(pristine.shape), dtype=torch.float32, pin_memory=True)   # this rank's columns
        a_host.copy_(pristine.cpu())
        ab_host = torch.empty((n, b + 1), dtype=torch.float32, pin_memory=True)
        e2e_ms = []
        for _ in range(args.e2e_steps + 1):
            torch.cuda.synchronize()
            torch.distributed.barrier()
            t0 = time.perf_counter()
            a.copy_(a_host, non_blocking=True)
            run_step()
            if rank == 0:
                ab_host.copy_(ab, non_blocking=True)
            torch.cuda.synchronize()
            dt = torch.tensor([(time.perf_counter() - t0) * 1e3], device=a.device)
            torch.distributed.all_reduce(dt, op=torch.distributed.ReduceOp.MAX)
            e2e_ms.append(float(dt.item()))
        e2e_ms = e2e_ms[1:]
        e2e = {"value": eff_tflops(n, statistics.median(e2e_ms) / 1e3), "unit": "TFLOP/s",
               "h2d_bytes_per_step": 4 * n * n, "d2h_bytes_per_step": 4 * n * (b + 1),
               "ms_per_step": statistics.median(e2e_ms), "steps": args.e2e_steps,
               "note": "Handle.reduce_dist: each rank's pinned host columns -> its GPU, reduce across ranks, "
                       "band -> host (rank 0)"}
        del a_host
    elif args.e2e_steps > 0:
        a_host = torch.empty((n, n), dtype=torch.float32, pin_memory=True)
        a_host.copy_(pristine.cpu())   # same input bits (device generator == workloads generator)
        ab_host = torch.empty((n, b + 1), dtype=torch.float32, pin_memory=True)
        h.reduce_host(a_host, b, nb, mode=mode, ab=ab_host)   # warm-up of the device copies
        e2e_ms = []
        for _ in range(args.e2e_steps):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            h.reduce_host(a_host, b, nb, mode=mode, ab=ab_host)
            e2e_ms.append((time.perf_counter() - t0) * 1e3)
        e2e_t = max(e2e_ms) if world == 1 else max(e2e_ms)
        e2e = {"value": eff_tflops(n, statistics.median(e2e_ms) / 1e3), "unit": "TFLOP/s",
               "h2d_bytes_per_step": 4 * n * n, "d2h_bytes_per_step": 4 * n * (b + 1),
               "ms_per_step": statistics.median(e2e_ms), "steps": args.e2e_steps,
               "note": "sbr_reduce_host: pinned host A -> device, reduce, band -> host (the paper's EVD "
                       "pipeline moves only the band, P:415)"}
        del a_host
    cpu = None
    if rank == 0 and not args.no_cpu_baseline:
        a_np = pristine.cpu().numpy()   # the same input bits
        cpu = cpu_oracle_sample(n, b, a_np, args.cpu_sample_s)
        cpu.pop("seconds_extrapolated", None)
        del a_np
    lapack = None
    if rank == 0 and not args.no_cpu_baseline and args.lapack_n > 0:
        try:
            lapack = lapack_sy2sb_baseline(min(args.lapack_n, n), b, n, seed)
        except Exception as e:  # pragma: no cover
            lapack = {"error": str(e)}

    if rank == 0:
        line = {
            "metric": METRIC,
            "value": value,
            "unit": "TFLOP/s",
            "n_gpus": world,
            "scaling": "strong",   # one matrix at any N (N = 1 included: the SCALE run divides the same work)
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": ms_per_step,
            "seconds_per_step": ms_per_step / 1e3,
            "higher_is_better": True,
            "vs_baseline": None,
            "dtype": {"3xtf32": "f32", "bf16": "bf16"}.get(mode, "f16"),
            "data": "synthetic",
            "config": {"workload": f"{cfg_name}: n={n} {input_desc}, b={b}, nb={nb}, "
                                   f"{ {'fp16': 'FP16-in/FP32-acc', 'bf16': 'BF16-in/FP32-acc (ablation)'}.get(mode, '3xTF32')}",
                       "n": n, "b": b, "nb": nb, "mode": mode,
                       "parallelism": f"sbr_reduce_dist over {world} GPUs: 1D block-cyclic nb-column blocks "
                                      f"(owner factors its panels; pass and SYR2K on own columns; NCCL "
                                      f"broadcast W_t / Y, all-reduce X_t)" if world > 1 else "single",
                       "l2": f"inputs {4 * n * n / 2**30:.1f} GiB >> 126 MB L2 (no flush needed)"},
            "frac_of_peak": {"fp16_spec_2250": value / world / 2250.0,
                             "fp16_measured": value / world / peaks.get("bf16_tflops", 1642.5),
                             "composite_roofline_model_ms": 88.4 if (n, b, nb) == (32768, 32, 1024) else None},
            "roofline": roof,
            "breakdown": breakdown,
            "cpu_baseline": cpu,
            "lapack_baseline": lapack,
            "e2e": e2e,
            "form_q": formq,
            "gpu_launches": launches,
            "clocks": clk.summary(),
            "step_ms": step_ms,
        }
        print(json.dumps(line), flush=True)
    h.close()
    if world > 1:
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
