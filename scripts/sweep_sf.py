"""In-process sweep of launch-time tunables of the sync-free triangles
(SPTRSV_SF_CTAS, SPTRSV_SF_BACKOFF are read at every solve): one analysis,
then per setting 5 profiled solves (L2 flushed); prints per-segment means.

    python scripts/sweep_sf.py C3 "SPTRSV_SF_CTAS=148" "SPTRSV_SF_CTAS=37,SPTRSV_SF_BACKOFF=0" ...
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_lun020_b200 as sp  # noqa: E402
from oracle import numeric as on  # noqa: E402
from workloads import generators as g  # noqa: E402


def main():
    cfg = sys.argv[1]
    nrhs = int(os.environ.get("SWEEP_NRHS", "1"))
    M = g.gen_matrix(cfg)
    b = g.gen_rhs(M.n, nrhs, seed=g.config_seed(cfg))
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, graphs=False)
    segs = plan.segments()
    cols = [0, nrhs // 2, nrhs - 1] if nrhs > 1 else [0]
    ref = on.solve(M, b[cols], threads=len(cols))
    B = torch.from_numpy(b[0]).cuda() if nrhs == 1 else torch.from_numpy(b).cuda().T
    X = torch.empty_like(B)
    flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
    base = dict(os.environ)
    for setting in [""] + sys.argv[2:]:
        os.environ.clear()
        os.environ.update(base)
        for kv in filter(None, setting.split(",")):
            k, v = kv.split("=")
            os.environ[k] = v
        for _ in range(2):
            sp.sptrsv_solve(plan, B, X)
        plan.set_profiling(True)
        acc = []
        for _ in range(5):
            flush.zero_()
            sp.sptrsv_solve(plan, B, X)
            acc.append(plan.seg_times())
        plan.set_profiling(False)
        torch.cuda.synchronize()
        t = np.mean(acc, axis=0)
        xh = X.cpu().numpy()
        err = on.rel_err(xh[None] if nrhs == 1 else xh.T[cols], ref)
        tri = sum(t[1 + i] for i, s in enumerate(segs) if s["kind"] == "TRI")
        sq = sum(t[1 + i] for i, s in enumerate(segs) if s["kind"] == "SQ")
        print(f"{setting or 'default':45s} total {t.sum():.3f} ms tri {tri:.3f} sq {sq:.3f} err {err:.1e} | "
              + " ".join(f"{v:.3f}" for v in t[1:-1]), flush=True)
    plan.free()


if __name__ == "__main__":
    main()
