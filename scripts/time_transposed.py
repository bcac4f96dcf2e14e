"""A^T x = b two ways (R31 / R32): a second plan analysed for A^T
(opts.transpose, pull-form kernels) vs the transposed sweep over A's own plan
(sptrsv_solve_transposed, push form, Alg 3).  Preprocessing (host CSR) and
solve (median of 10, L2 flushed) per config; parity vs the oracle on the
explicitly transposed matrix.  Prints one JSON line per config.

    python scripts/time_transposed.py C2 C3 C4 [--out profiles/r02_transposed.json]
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icpp_lun020_b200 as sp  # noqa: E402
from oracle import numeric as on  # noqa: E402
from workloads import generators as g  # noqa: E402


def timed(fn, flush, reps=10):
    for _ in range(3):
        fn()
    ts = []
    for _ in range(reps):
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    out = sys.argv[sys.argv.index("--out") + 1] if "--out" in sys.argv else None
    if out in args:
        args.remove(out)
    flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
    res = []
    for cfg in args or ["C2", "C3", "C4"]:
        M, b = g.gen_config(cfg, nrhs=1)
        B = torch.from_numpy(b[0]).cuda()
        X = torch.empty_like(B)
        ref = on.solve(g.transpose(M), b)
        rec = {"config": cfg, "n": M.n, "nnz": M.nnz}
        for mode in ("second_plan", "same_plan"):
            t0 = time.perf_counter()
            plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, transpose=(mode == "second_plan"))
            torch.cuda.synchronize()
            pre = (time.perf_counter() - t0) * 1e3
            if mode == "second_plan":
                fn = lambda: sp.sptrsv_solve(plan, B, X)  # noqa: E731
            else:
                fn = lambda: sp.sptrsv_solve(plan, B, X, transposed=True)  # noqa: E731
            ms = timed(fn, flush)
            err = on.rel_err(X.cpu().numpy()[None], ref)
            rec[mode] = {"preprocess_ms": pre, "solve_ms": ms, "gflops": 2 * M.nnz / ms / 1e6, "rel_err": err,
                         "plan_device_bytes": plan.info().get("device_bytes")}
            plan.free()
        print(json.dumps(rec), flush=True)
        res.append(rec)
    if out:
        json.dump(res, open(out, "w"), indent=1)


if __name__ == "__main__":
    main()
