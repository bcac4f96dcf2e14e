#!/usr/bin/env python
"""Benchmark of the recursive-block SpTRSV on B200 (BASELINE.json metric:
"SpTRSV solve GFLOPS (2*nnz/t) and HBM GB/s % of peak; preprocess ms").

One step = one sptrsv_solve of the whole hot path (permute-in, every triangle
and square segment of Alg 7, permute-out) over one RHS batch of the workload.
Default workload at one GPU: C3 = BASELINE.json configs[2], the largest
single-RHS configuration (layered power-law L, n = 4M, ~81M nnz, 2,815
levels; mirrors vas_stokes_4M).  Inputs are resident in HBM
when the timed region starts; L2 (126 MB) is flushed between timed solves
with a 256 MB write.  Repeated solves with the same buffers replay a CUDA
graph captured by the library (opts.graphs): the timed region holds no host
synchronisation; per-segment times come from a separate attribution pass
(profiling on, kernels launched one by one) after it.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3] [--impl ours|reference]

Multi-GPU (torchrun, one process per GPU): the default workload becomes C5,
whose 512 RHS columns are sharded over the ranks (the only
config whose solve shards); the plan is replicated and there is no collective
on the timed data path.  An explicit --config C1..C4 runs one independent
replica per rank instead ("replicas only").
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "SpTRSV solve GFLOPS (2*nnz*nrhs/t)"
DEFAULT_NRHS = {"C1": 1, "C2": 1, "C3": 1, "C4": 1, "C5": 512}
WORKLOAD = {
    "C1": "C1 random lower triangle n=1000 ~5 nnz/row fp64",
    "C2": "C2 IC(0) factor of 2D 5-point Laplacian 1000x1000 (n=1M, nnz=2.998M) fp64",
    "C3": "C3 layered power-law L n=4M ~20 nnz/row 2815 levels fp64",
    "C4": "C4 supernodal factor n=500K w=64 dense tiles fp64",
    "C5": "C5 random L n=2M ~10 nnz/row, 512 RHS fp64",
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default=None, help="C1..C5; default C3 at 1 GPU, C5 (sharded) at N > 1")
    ap.add_argument("--nrhs", type=int, default=None)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--selector", default="B200", choices=["B200", "PAPER"])
    ap.add_argument("--variant", default="REC", choices=["REC", "COL", "ROW"])
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    ap.add_argument("--no-flush", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=10.0, help="oracle baseline budget")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--transpose", action="store_true",
                    help="solve A^T x = b from the workload's A (opts.transpose, DESIGN.md R31)")
    ap.add_argument("--dist", action="store_true",
                    help="run the NCCL sharded multi-RHS path even at world size 1 (tests the code path)")
    return ap.parse_args()


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self._stop = threading.Event()
        self._t = None

    def _run(self):
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True,
                                     timeout=5).stdout.strip()
                if out:
                    self.rows.append([v.strip() for v in out.split(",")])
            except Exception:
                pass
            self._stop.wait(0.2)

    def start(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()

    def wait_first(self, timeout: float = 3.0):
        """Block until the first sample landed: the first nvidia-smi call
        (process start + driver queries) then falls before the timed steps,
        where it made the first step of short runs an outlier."""
        t0 = time.time()
        while not self.rows and time.time() - t0 < timeout:
            time.sleep(0.01)

    def stop(self):
        self._stop.set()
        if self._t:
            self._t.join(timeout=10)
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for nm, v in zip(names, r[5:9]):
                if v.strip().lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows)}


def algorithmic_bytes(n, nnz, nrhs, vb):
    """Compulsory traffic of any CSR SpTRSV: read L once,
    read b once, write x once."""
    return nnz * (vb + 4) + 4 * (n + 1) + 2 * n * nrhs * vb


def seg_alg_bytes(seg, nrhs, vb):
    """Algorithmic bytes of one segment launch: its matrix
    entries (value + column), its row pointers, and its vector traffic."""
    m = seg["row1"] - seg["row0"]
    if seg["kind"] == "TRI":
        off = seg["nnz"] - m
        return off * (vb + 4) + (m + 1) * 4 + m * vb + 2 * m * nrhs * vb  # + diag, b in, x out
    nz = seg["nnz"]
    rows = m - seg["empty_rows"]
    ncols = seg["col1"] - seg["col0"]
    return nz * (vb + 4) + (rows + 1) * 4 + ncols * nrhs * vb + 2 * rows * nrhs * vb


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


def load_traffic(kernel_impl: str):
    """dram bytes per launch of the dominant kernel ("<config>:<impl>") from
    the committed ncu summary (profiles/ncu_summary.json), else None."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        d = json.load(open(p))
        return d.get("dram_bytes_per_launch", {}).get(kernel_impl)
    except Exception:
        return None


def cpu_baseline(M, b, budget_s):
    """Oracle (Alg 1, plain C, fp64) on the host, 1 thread per RHS column
    group; repeated full solves until ~budget_s of CPU work (bounded sample)."""
    from oracle import numeric as on
    nrhs = b.shape[0]
    threads = 1 if nrhs == 1 else min(nrhs, len(os.sched_getaffinity(0)))
    if nrhs > 1:
        # bounded sample: the first columns only, as many as threads x 2
        cols = min(nrhs, threads * 2)
        bs = np.ascontiguousarray(b[:cols])
    else:
        cols, bs = 1, b
    x, dt, used = on.solve_timed(M, bs, threads=threads)
    reps, tot = 1, dt
    while tot < budget_s and reps < 10000:
        _, dt, used = on.solve_timed(M, bs, threads=threads)
        tot += dt
        reps += 1
    per = tot / reps
    gflops = 2.0 * M.nnz * cols / per / 1e9
    sample = (f"{reps} full solves of the workload matrix x {cols} of {nrhs} RHS column(s), "
              f"{tot:.1f} s of CPU time")
    return {"value": gflops, "unit": "GFLOPS", "cores": used, "kind": "oracle", "sample": sample,
            "cpu_model": cpu_model(), "ms_per_solve": per * 1e3}


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def default_config(args):
    if args.config is None:
        ws, _, _ = dist_env()
        args.config = "C5" if (ws > 1 or args.dist) else "C3"
    return args.config


def run_reference(args):
    """--impl reference: the oracle, as it stands, timed on the host cores."""
    default_config(args)
    ws, rank, _ = dist_env()
    if rank != 0:
        return
    from workloads import generators as g
    from oracle import numeric as on
    nrhs = args.nrhs or DEFAULT_NRHS[args.config]
    M = g.gen_matrix(args.config)
    threads = 1 if nrhs == 1 else min(nrhs, len(os.sched_getaffinity(0)))
    cols = nrhs if nrhs == 1 else min(nrhs, threads * 2)
    bs = g.gen_rhs_cols(M.n, 0, cols, seed=g.config_seed(args.config))  # a bounded sample of the columns
    for _ in range(args.warmup):
        on.solve_timed(M, bs, threads=threads)
    ts = []
    for _ in range(args.steps):
        _, dt, used = on.solve_timed(M, bs, threads=threads)
        ts.append(dt)
    t = float(np.mean(ts))
    val = 2.0 * M.nnz * cols / t / 1e9
    line = {"metric": METRIC, "value": val, "unit": "GFLOPS", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
            "config": {"workload": WORKLOAD[args.config], "n": M.n, "nnz": M.nnz, "nrhs": nrhs, "nrhs_timed": cols},
            "cpu_baseline": {"value": val, "unit": "GFLOPS", "cores": used, "kind": "oracle",
                             "cpu_model": cpu_model(),
                             "sample": f"{args.steps} full solves x {cols} RHS column(s)"},
            "e2e": {"value": val, "unit": "GFLOPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def load_tlvl():
    """Measured per-level synchronisation latencies (scripts/microbench/t_lvl.cu,
    summarised in profiles/t_lvl.json), or None."""
    p = os.path.join(ROOT, "profiles", "t_lvl.json")
    try:
        return json.load(open(p))
    except Exception:
        return None


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    import torch.distributed as dist

    default_config(args)
    ws, rank, local = dist_env()
    use_dist = ws > 1 or args.dist
    if use_dist:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29517")
        dist.init_process_group("nccl", device_id=torch.device("cuda", local), rank=rank, world_size=ws)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)

    import paper_conf_icpp_lun020_b200 as sp
    from paper_conf_icpp_lun020_b200.dist import check_replicated, dist_solve, shard_bounds
    from workloads import generators as g

    cfg = args.config
    nrhs_total = args.nrhs or DEFAULT_NRHS[cfg]
    # C5 (multi-RHS) shards its RHS columns over the ranks (strong scaling);
    # every other config runs one independent replica per rank (weak scaling,
    # a single solve does not shard)
    sharded = nrhs_total > 1 and use_dist
    if sharded:
        c0, c1 = shard_bounds(nrhs_total, ws, rank)
    else:
        c0, c1 = 0, nrhs_total
    nrhs = c1 - c0
    tdt = torch.float64 if args.dtype == "f64" else torch.float32
    npdt = np.float64 if args.dtype == "f64" else np.float32
    vb = 8 if args.dtype == "f64" else 4
    M = g.gen_matrix(cfg)
    seed = g.config_seed(cfg) if (sharded or rank == 0) else g.config_seed(cfg) + 7919 * rank
    b_np = g.gen_rhs_cols(M.n, c0, c1, seed=seed)  # (nrhs, n): this rank's columns
    val = M.val if args.dtype == "f64" else M.val.astype(np.float32)

    # preprocess (analysis + upload, median of 3 after one
    # warm-up).  The CSR resident on the device runs the device analysis
    # (f-2, analyse_dev.cu); a host CSR runs the host analysis + upload.
    kw = dict(selector=args.selector, variant=args.variant, transpose=args.transpose)
    dcsr = [torch.from_numpy(a).to(dev) for a in (M.row_ptr, M.col_idx, val)]
    torch.cuda.synchronize()

    def time_analyse(src, **extra):
        ts = []
        for i in range(4):
            t0 = time.perf_counter()
            p2 = sp.sptrsv_analyse(*src, **kw, **extra)
            torch.cuda.synchronize()
            if i:
                ts.append((time.perf_counter() - t0) * 1e3)
            where = p2.info()["analysis"]
            p2.free()
        return float(np.median(ts)), where

    preprocess_ms, analysis_where = time_analyse(dcsr)
    preprocess_host_ms, _ = time_analyse((M.row_ptr, M.col_idx, val))
    plan = sp.sptrsv_analyse(*dcsr, **kw)
    del dcsr
    info = plan.info()
    segs = plan.segments()
    if use_dist:
        check_replicated(plan)

    B = torch.from_numpy(b_np).to(dev, tdt).T  # (n, nrhs) column-major
    if nrhs == 1:
        B = B[:, 0].contiguous()
    X = torch.empty_like(B)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream(dev)

    assert args.warmup >= 3, "W >= 3: the 2nd solve captures the CUDA graph, the timed ones replay it"
    # clocks are sampled from before the warm-up to the end of the timed
    # region (every 0.2 s); the first sample is taken before any solve
    clocks = ClockSampler(local)
    clocks.start()
    clocks.wait_first()
    for _ in range(args.warmup):
        if not args.no_flush:
            flush.zero_()
        sp.sptrsv_solve(plan, B, X, stream=stream)
    torch.cuda.synchronize()

    # ---------------- timed region: K solves (graph replays), CUDA events on
    # the solve stream, no host synchronisation between steps
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    for i in range(args.steps):
        if not args.no_flush:
            flush.zero_()
        starts[i].record(stream)
        sp.sptrsv_solve(plan, B, X, stream=stream)
        ends[i].record(stream)
    torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    clk = clocks.stop()
    step_ms = np.array([s.elapsed_time(e) for s, e in zip(starts, ends)])
    t_local = float(np.sum(step_ms)) / 1e3
    if ws > 1:
        tt = torch.tensor([t_local], dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_max = float(tt.item())
    else:
        t_max = t_local

    # warm solves (L2 not flushed; the paper's back-to-back average, L316)
    warm = []
    for _ in range(min(args.steps, 20)):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        sp.sptrsv_solve(plan, B, X, stream=stream)
        e1.record(stream)
        warm.append((e0, e1))
    torch.cuda.synchronize()
    warm_ms = np.array([a.elapsed_time(b2) for a, b2 in warm])

    # ---------------- attribution pass: per-segment CUDA events (profiling
    # launches the kernels one by one and reads the events after each solve)
    plan.set_profiling(True)
    seg_acc = None
    nattr = min(args.steps, 20)
    for i in range(nattr):
        if not args.no_flush:
            flush.zero_()
        sp.sptrsv_solve(plan, B, X, stream=stream)
        st = plan.seg_times()
        seg_acc = st if seg_acc is None else seg_acc + st
    plan.set_profiling(False)
    torch.cuda.synchronize()

    # whole-job work per step: all RHS columns (sharded) or one replica per rank
    flops_job = 2.0 * M.nnz * (nrhs_total if sharded else nrhs * ws)
    value = flops_job * args.steps / t_max / 1e9
    ms_per_step = t_max / args.steps * 1e3
    timing = {"mean_ms": float(step_ms.mean()), "median_ms": float(np.median(step_ms)),
              "p90_ms": float(np.percentile(step_ms, 90)), "min_ms": float(step_ms.min()),
              "warm_mean_ms": float(warm_ms.mean()), "warm_median_ms": float(np.median(warm_ms)),
              "warm_p90_ms": float(np.percentile(warm_ms, 90)),
              "graph_replay": True,
              "segment_pass": f"{nattr} separate solves, profiling on (no graph), L2 flushed"}

    # ---------------- roofline of the dominant kernel
    peak, peak_kind = load_peaks()
    seg_mean = seg_acc / nattr  # [perm-in, seg..., perm-out]
    def run_impl(sg):
        """The kernel family that actually runs the segment at this nrhs: the
        plan's impl for one RHS; with many RHS squares run the SpMM (sq_multi)
        and the wave triangles the multi-RHS sync-free kernel; supernodal
        triangles run tri_supernode_multi from 16 RHS (exec.cu kSnMultiMinRhs)."""
        if nrhs == 1:
            return sg["impl"]
        if sg["kind"] == "SQ":
            return "SQ_SPMM"
        if sg["impl"] == "TRI_SUPERNODE" and nrhs >= 16 and not os.environ.get("SPTRSV_NO_SN_MULTI"):
            return "TRI_SUPERNODE_MULTI"
        return {"TRI_SUPERNODE": "TRI_SYNCFREE", "TRI_PIPE": "TRI_SYNCFREE"}.get(sg["impl"], sg["impl"])

    names = ["permute_in"] + [f"seg{i}:{run_impl(s)}" for i, s in enumerate(segs)] + ["permute_out"]
    dom = int(np.argmax(seg_mean))
    dep = None
    if 1 <= dom <= len(segs):
        dseg = segs[dom - 1]
        dbytes = seg_alg_bytes(dseg, nrhs, vb)
        dimpl = run_impl(dseg)
        # a dependency floor applies to a one-RHS triangle solved row by row
        # (the supernodal kernels take one hop per piece of up to 32 rows, and
        # many-RHS triangles are bound by their X-row gathers, DESIGN 5.7)
        if dseg["kind"] == "TRI" and dseg["nlevels"] > 1 and nrhs == 1 and not dimpl.startswith("TRI_SUPERNODE"):
            ns_lvl = seg_mean[dom] * 1e6 / dseg["nlevels"]
            dep = {"nlevels": dseg["nlevels"], "ns_per_level": ns_lvl}
            tl = load_tlvl()
            if tl:
                # the floor of ONE dependent level for the kernel family: an
                # on-SM barrier chain for the single-SM / one-cluster kernels,
                # a cross-SM store -> poll hop through L2 for the multi-SM ones
                on_sm = dimpl in ("TRI_CHAIN", "TRI_PIPE")
                fl = tl.get("smem_chain_bar_ns") if on_sm else tl.get("cross_sm_hop_ns")
                dep["t_lvl_floor_ns"] = fl
                dep["floor_frac"] = fl / ns_lvl if fl else None
                dep["t_lvl_source"] = ("profiles/t_lvl.json: " + ("bar.sync + ld.shared/DFMA/st.shared chain, 1 SM"
                                       if on_sm else "cross-SM flag ping-pong through L2 (st/ld.relaxed.gpu)"))
    else:
        dbytes = M.n * 4 + 2 * M.n * nrhs * vb
        dimpl = "PERMUTE"
    achieved = dbytes / (seg_mean[dom] / 1e3) / 1e9
    # the committed capture is per (config, kernel) at the config's default
    # RHS count; other RHS counts carry their own key ("C4:...@64")
    tr = load_traffic(f"{cfg}:{dimpl}" + (f"@{nrhs}" if nrhs_total != DEFAULT_NRHS[cfg] else ""))
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": tr, "kernel": names[dom], "share_of_step": float(seg_mean[dom] / seg_mean.sum()),
                "alg_bytes_per_launch": dbytes,
                "peak_source": f"{peak_kind} copy bandwidth (MEASURED_PEAKS.json hbm_gbs)"}
    if dep:
        roofline["dependency"] = dep
    whole_bytes = algorithmic_bytes(M.n, M.nnz, nrhs, vb)
    whole = {"achieved_gbs": whole_bytes / (ms_per_step / 1e3) / 1e9,
             "frac": whole_bytes / (ms_per_step / 1e3) / 1e9 / peak, "alg_bytes": whole_bytes}

    # ---------------- end to end through the public API with host buffers
    e2e_iters = max(3, min(args.steps, 20 if nrhs_total == 1 else 3))
    if sharded:
        # root: pinned host B (all columns) -> H2D -> dist_solve (NCCL scatter,
        # per-rank solve, NCCL gather) -> D2H; max over ranks
        if rank == 0:
            b_all = g.gen_rhs(M.n, nrhs_total, seed=g.config_seed(cfg), dtype=npdt)
            Bh = torch.from_numpy(b_all).pin_memory()  # (k, n) row-major == (n, k) column-major
            Xh = torch.empty_like(Bh).pin_memory()
            del b_all
        e2e_ms = []
        for it in range(e2e_iters + 1):
            dist.barrier()
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            Bd = Bh.to(dev, non_blocking=True).T if rank == 0 else None
            Xd = dist_solve(plan, Bd, nrhs=None if rank == 0 else nrhs_total)
            if rank == 0:
                Xh.copy_(Xd.T, non_blocking=True)
            e1.record(stream)
            e1.synchronize()
            if it:
                e2e_ms.append(e0.elapsed_time(e1))
            del Bd, Xd
        h2d = d2h = M.n * nrhs_total * vb
    else:
        Bh = torch.from_numpy(b_np.astype(npdt)).pin_memory().T
        if nrhs == 1:
            Bh = Bh[:, 0].contiguous().pin_memory()
        Xh = torch.empty_like(Bh).pin_memory() if nrhs == 1 else torch.empty(nrhs, M.n, dtype=tdt).pin_memory().T
        for _ in range(2):
            sp.sptrsv_solve(plan, Bh, Xh, stream=stream)
        e2e_ms = []
        for _ in range(e2e_iters):
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            sp.sptrsv_solve(plan, Bh, Xh, stream=stream)  # H2D + solve + D2H (+ sync)
            e1.record(stream)
            e1.synchronize()
            e2e_ms.append(e0.elapsed_time(e1))
        h2d = d2h = M.n * nrhs * vb
    e2e_t = float(np.mean(e2e_ms)) / 1e3
    if ws > 1:
        tt = torch.tensor([e2e_t], dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        e2e_t = float(tt.item())
    e2e = {"value": flops_job / e2e_t / 1e9, "unit": "GFLOPS", "h2d_bytes_per_step": h2d,
           "d2h_bytes_per_step": d2h, "ms_per_step": e2e_t * 1e3,
           "path": "dist_solve (NCCL scatter/gather) from pinned host B on rank 0" if sharded
           else ("sptrsv_solve with pinned host b/x (column blocks: H2D / solve / D2H overlapped on three "
                 "streams inside the call)" if nrhs >= 32 else
                 "sptrsv_solve with pinned host b/x (H2D + solve + D2H inside the call)")}

    # ---------------- parity of the timed result (sampled for multi-RHS)
    parity = None
    if rank == 0:
        from oracle import numeric as on
        cols = list(range(nrhs))  # every column of the timed result
        xs = X.double().cpu().numpy()
        xs = xs[None] if xs.ndim == 1 else xs.T[cols]
        ref = on.solve(g.transpose(M) if args.transpose else M, b_np[cols],
                       threads=max(1, min(len(cols), len(os.sched_getaffinity(0)))))
        errs = [on.rel_err(xs[c], ref[c]) for c in range(len(cols))]
        parity = {"rel_err": float(max(errs)), "tol": 1e-10 if vb == 8 else 1e-4,
                  "columns_checked": len(cols), "of_columns": nrhs}

    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(g.transpose(M) if args.transpose else M, b_np, args.cpu_seconds)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "GFLOPS", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": "strong" if sharded or (nrhs_total > 1 and ws == 1) else "weak",
            "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            "config": {"workload": WORKLOAD[cfg], "n": M.n, "nnz": M.nnz, "nrhs": nrhs_total,
                       "nrhs_per_rank": nrhs, "selector": args.selector, "variant": args.variant,
                       "op": "A^T x = b" if args.transpose else "A x = b",
                       "depth": info["depth"], "segments": len(segs),
                       "l2": "flushed (256 MB write) between timed solves" if not args.no_flush else "not flushed",
                       "parallelism": (f"rhs-columns sharded x{ws} (NCCL scatter/gather only in e2e)" if sharded
                                       else f"rhs-replicas x{ws}")},
            "preprocess_ms": preprocess_ms,
            "preprocess": {
                "device_csr_ms": preprocess_ms,
                "analysis": ["host", "device", "device levels/reorder + host formats"][analysis_where],
                "host_csr_ms": preprocess_host_ms,
                "over_solve": preprocess_ms / ms_per_step,
                # Table 5: preprocessing + k solves, and the
                # share of preprocessing in it
                "amortised": {str(k): {"total_ms": preprocess_ms + k * ms_per_step,
                                       "pre_share": preprocess_ms / (preprocess_ms + k * ms_per_step)}
                              for k in (1, 100, 500, 1000)},
            },
            "hbm_whole_solve": whole,
            "roofline": roofline,
            "timing": timing,
            "segment_ms": {nm: float(v) for nm, v in zip(names, seg_mean)},
            "e2e": e2e,
            "gpu_launches": int(info["launches_per_solve"]) * args.steps,
            "clocks": clk,
            "parity": parity,
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    if use_dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
