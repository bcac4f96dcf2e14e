"""Per-level timeline of the sync-free triangles of one solve (debug tool).

Needs a library built with -DSPTRSV_SF_TRACE (SPTRSV_NVCC_FLAGS) and the
SPTRSV_SF_TRACE=<dir> environment variable: every row stores its claim and
completion %globaltimer stamps.  For each sync-free triangle this prints the
per-level critical path split into
  claim-late : the level's last row was claimed after its last dependency
               had completed (the grid / ticket order is the limiter),
  detect     : completion of the last row minus the completion of its
               latest dependency (poll detection + compute + store),
and the mean level time.

    SPTRSV_SF_TRACE=/tmp python scripts/sf_trace.py C3
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_lun020_b200 as sp  # noqa: E402
from workloads import generators as g  # noqa: E402


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
    d = os.environ["SPTRSV_SF_TRACE"]
    M = g.gen_matrix(cfg)
    b = g.gen_rhs(M.n, 1, seed=g.config_seed(cfg))
    plan = sp.sptrsv_analyse(M.row_ptr, M.col_idx, M.val, graphs=False)
    B = torch.from_numpy(b[0]).cuda()
    for _ in range(3):
        X = sp.sptrsv_solve(plan, B)
    torch.cuda.synchronize()
    plan.set_profiling(True)
    X = sp.sptrsv_solve(plan, B)
    times = plan.seg_times()
    tr = np.fromfile(os.path.join(d, "sf_trace.bin"), dtype=np.uint64).reshape(-1, 2).astype(np.int64)
    segs = plan.segments()
    rp, ci, _ = plan.matrix()
    lev = plan.levels()
    for i, s in enumerate(segs):
        if s["kind"] != "TRI" or s["impl"] != "TRI_SYNCFREE":
            continue
        r0, r1 = s["row0"], s["row1"]
        cl, dn = tr[r0:r1, 0], tr[r0:r1, 1]
        if not np.all(dn > 0):
            print(f"seg{i}: missing stamps ({np.sum(dn == 0)} rows)")
            continue
        t0 = cl.min()
        cl, dn = cl - t0, dn - t0
        L = lev[r0:r1]
        nl = int(L.max()) + 1
        lvl_done = np.full(nl, -1, np.int64)
        np.maximum.at(lvl_done, L, dn)
        crit = np.zeros(nl, np.int64)
        order = np.lexsort((dn, L))  # last row of each level = last in its group
        ends = np.searchsorted(L[order], np.arange(nl), side="right") - 1
        crit = order[ends]
        claim_late = detect = 0.0
        det = []
        late = 0
        for l in range(1, nl):
            c = crit[l]
            r = r0 + c
            cols = ci[rp[r]:rp[r + 1] - 1]
            cols = cols[cols >= r0] - r0
            dep_done = dn[cols].max() if cols.size else 0
            if cl[c] > dep_done:
                late += 1
                claim_late += cl[c] - dep_done
            det.append(dn[c] - max(dep_done, cl[c]))
        det = np.array(det)
        total = dn.max()
        print(f"seg{i}: rows {r1 - r0} levels {nl} span {total / 1e3:.1f} us (event {times[1 + i] * 1e3:.1f} us) "
              f"per level {total / nl:.0f} ns | claim-late levels {late} ({claim_late / 1e3:.1f} us) | "
              f"detect mean {det.mean():.0f} ns p10 {np.percentile(det, 10):.0f} p50 {np.median(det):.0f} "
              f"p90 {np.percentile(det, 90):.0f} | "
              f"row claim->done p50 {np.median(dn - cl):.0f} ns")
        w = np.bincount(L, minlength=nl)
        dl = np.diff(lvl_done)
        big = np.argsort(dl)[-5:][::-1]
        print("   slowest level steps:", [(int(l + 1), int(dl[l]), int(w[l + 1])) for l in big])
        crit_deg = np.array([rp[r0 + c + 1] - rp[r0 + c] - 1 for c in crit])
        print("   critical-row degree p50/p90/max:", int(np.median(crit_deg)), int(np.percentile(crit_deg, 90)),
              int(crit_deg.max()))
    plan.free()


if __name__ == "__main__":
    main()
