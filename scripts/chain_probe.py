"""Per-level cost of the sync-free triangle kernels on synthetic layered
DAGs (debug tool): a pure chain (width 1) and layered DAGs of width w whose
rows depend on one row of the previous level plus k-1 older rows.  Prints
ns per level for each kernel variant (SPTRSV_SF_* env set per variant)."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_lun020_b200 as sp  # noqa: E402
from oracle import numeric as on  # noqa: E402
from workloads import generators as g  # noqa: E402


def layered(levels, w, k, seed=5):
    rng = np.random.default_rng(seed)
    n = levels * w
    rows, cols = [], []
    for l in range(1, levels):
        r = np.arange(l * w, (l + 1) * w)
        rows.append(r)
        cols.append(rng.integers((l - 1) * w, l * w, size=w))
        for _ in range(k - 1):
            rows.append(r)
            cols.append(rng.integers(0, l * w, size=w))
    rows = np.concatenate(rows)
    cols = np.concatenate(cols)
    return g._assemble(n, rows, cols, rng, f"layered{levels}x{w}k{k}")


def main():
    variants = {"V1": {}, "MIXED": {"SPTRSV_SF_MIXED": "1"}, "WROW": {"SPTRSV_SF_WROW": "1"}}
    cases = [("chain", layered(20000, 1, 1)), ("w64", layered(2000, 64, 2)), ("w650", layered(400, 650, 3)),
             ("w650k8", layered(400, 650, 8))]
    flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
    for name, M in cases:
        b = g.gen_rhs(M.n, 1, seed=3)
        ref = on.solve(M, b)
        B = torch.from_numpy(b[0]).cuda()
        line = []
        for vn, env in variants.items():
            for k2 in ("SPTRSV_SF_MIXED", "SPTRSV_SF_WROW"):
                os.environ.pop(k2, None)
            os.environ.update(env)
            plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, depth=0, reorder=False,
                                     force_tri_impl="TRI_SYNCFREE", graphs=False)
            nl = plan.segments()[0]["nlevels"]
            X = torch.empty_like(B)
            for _ in range(3):
                sp.sptrsv_solve(plan, B, X)
            plan.set_profiling(True)
            ts = []
            for _ in range(5):
                flush.zero_()
                sp.sptrsv_solve(plan, B, X)
                ts.append(plan.seg_times()[1])
            err = on.rel_err(X.cpu().numpy()[None], ref)
            line.append(f"{vn} {np.median(ts) * 1e6 / nl:6.0f} ns/level (err {err:.0e})")
            plan.free()
        print(f"{name:8s} n={M.n} levels={nl}: " + " | ".join(line), flush=True)


if __name__ == "__main__":
    main()
