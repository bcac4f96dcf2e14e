"""Structural oracle -- TEST INFRASTRUCTURE ONLY.

What the paper's preprocessing computes, step by step in the paper's order
(the readings of ambiguous passages are numbered as in
DESIGN.md section 3 "Readings"):

  1. levels of a triangular (sub)matrix            Alg 2
  2. level-set reordering of every triangle          Sec 3.3
  3. recursive split node(lo, hi, d)                 Alg 6
     with the depth rule
  4. column / row block variants on the same leaves  Alg 4/5, PAPER.md:L146-L176
  5. block contents taken from the final P L P^T     (reading R6)
  6. per-block features and Alg 7's decision tree    Sec 3.4

Plain numpy; the level sweep of step 1 runs in the oracle's plain C
(csrc/oracle.c: oracle_levels) and has a pure-Python Alg 2 peel-off twin
(``levels_peel``) for brute-force agreement on small inputs.
"""
from __future__ import annotations

import ctypes
import dataclasses

import numpy as np

from .numeric import lib as _clib

# kernel labels (Alg 7) -- numbering is the oracle's own; the test maps the
# library's enum onto these names explicitly
TRI_COMPLETELY_PARALLEL = "COMPLETELY_PARALLEL"
TRI_LEVEL_SET = "LEVEL_SET"
TRI_SYNC_FREE = "SYNC_FREE"
TRI_NEAR_SERIAL = "NEAR_SERIAL"  # the cuSPARSE role of Alg 7 (L256, reading R14)
SQ_SCALAR_CSR = "SCALAR_CSR"
SQ_SCALAR_DCSR = "SCALAR_DCSR"
SQ_VECTOR_CSR = "VECTOR_CSR"
SQ_VECTOR_DCSR = "VECTOR_DCSR"


# ---------------------------------------------------------------------------
# 1. levels
# ---------------------------------------------------------------------------
def levels_sweep(m: int, row_ptr: np.ndarray, col_idx: np.ndarray) -> tuple[np.ndarray, int]:
    """level[i] = 0 if row i has no off-diagonal (col < i) entry, else
    1 + max(level[j]) over them; nlevels = max+1 (reading R5: only entries
    inside the given triangle count).  Local CSR indices 0..m-1."""
    rp = np.ascontiguousarray(row_ptr, dtype=np.int64)
    ci = np.ascontiguousarray(col_idx, dtype=np.int32)
    lev = np.zeros(m, dtype=np.int32)
    if m == 0:
        return lev, 0
    nl = _clib().oracle_levels(m, rp.ctypes.data_as(ctypes.c_void_p),
                               ci.ctypes.data_as(ctypes.c_void_p),
                               lev.ctypes.data_as(ctypes.c_void_p))
    return lev, int(nl)


def levels_peel(m: int, row_ptr, col_idx) -> tuple[np.ndarray, int]:
    """Algorithm 2's PREPROCESS-LEVELSET as written: in
    round li, every not-yet-assigned component whose dependencies are all
    assigned (to earlier rounds) joins level li.  Pure Python; small m."""
    deps = [[int(j) for j in col_idx[row_ptr[i]:row_ptr[i + 1]] if j < i] for i in range(m)]
    lev = [-1] * m
    li = 0
    left = m
    while left:
        ready = [i for i in range(m) if lev[i] < 0 and all(0 <= lev[j] < li for j in deps[i])]
        assert ready, "cycle"
        for i in ready:
            lev[i] = li
        left -= len(ready)
        li += 1
    return np.array(lev, dtype=np.int32), li


def level_stats(level: np.ndarray, nlevels: int):
    """(min, avg, max) level size; avg = floor(n / nlevels) (Table 4 convention,
    PAPER.md:L326-L334)."""
    if nlevels == 0:
        return 0, 0, 0
    sizes = np.bincount(level, minlength=nlevels)
    return int(sizes.min()), int(level.size // nlevels), int(sizes.max())


# ---------------------------------------------------------------------------
# 3. depth rule (reading R2)
# ---------------------------------------------------------------------------
def depth_rule(n: int, min_block_rows: int) -> int:
    """Largest d >= 0 with d == 0 or floor(n / 2^d) >= min_block_rows:
    'constantly divide the matrix until the number of rows of the next
    smallest block is less than' the threshold."""
    assert min_block_rows >= 1
    d = 0
    while (n >> (d + 1)) >= min_block_rows:
        d += 1
    return d


def clamp_depth(n: int, depth: int) -> int:
    """A forced depth is clamped so the smallest block keeps >= 1 row
    (reading R1b)."""
    if n <= 1:
        return 0
    return min(depth, n.bit_length() - 1)


def paper_threshold(cuda_cores: int) -> int:
    """20 x #CUDA cores (20 x 4608 = 92160 on Titan RTX)."""
    return 20 * cuda_cores


# ---------------------------------------------------------------------------
# 4. partition geometry (no matrix needed)
# ---------------------------------------------------------------------------
@dataclasses.dataclass
class Seg:
    kind: str  # "TRI" | "SQ"
    row0: int
    row1: int
    col0: int
    col1: int
    nnz: int = 0
    nlevels: int = 0
    nnz_per_row: int = 0
    empty_rows: int = 0
    kernel: str = ""
    format: str = ""


def rec_leaves(lo: int, hi: int, d: int, out: list):
    """Leaves of node(lo, hi, d): mid = lo + floor((hi-lo)/2) (reading R1)."""
    if d == 0:
        out.append((lo, hi))
        return
    mid = lo + (hi - lo) // 2
    rec_leaves(lo, mid, d - 1, out)
    rec_leaves(mid, hi, d - 1, out)


def partition(n: int, depth: int, variant: str) -> list[Seg]:
    """Segment geometry in execution order.

    REC (Alg 6): in-order TRI(top), SQ(rows [mid,hi) x cols [lo,mid)), TRI(bottom).
    COL (Alg 4, reading R16): TRI_k then RECT rows [e_k, n) x cols [s_k, e_k).
    ROW (Alg 5, reading R17): RECT rows [s_k, e_k) x cols [0, s_k) then TRI_k.
    All three use the same 2^d leaves (L182, reading R18).
    """
    segs: list[Seg] = []
    if n == 0:
        return segs
    if variant == "REC":
        def node(lo, hi, d):
            if d == 0:
                segs.append(Seg("TRI", lo, hi, lo, hi))
                return
            mid = lo + (hi - lo) // 2
            node(lo, mid, d - 1)
            segs.append(Seg("SQ", mid, hi, lo, mid))
            node(mid, hi, d - 1)
        node(0, n, depth)
        return segs
    leaves: list = []
    rec_leaves(0, n, depth, leaves)
    K = len(leaves)
    for k, (s, e) in enumerate(leaves):
        if variant == "COL":
            segs.append(Seg("TRI", s, e, s, e))
            if k != K - 1:
                segs.append(Seg("SQ", e, n, s, e))
        elif variant == "ROW":
            if k != 0:
                segs.append(Seg("SQ", s, e, 0, s))
            segs.append(Seg("TRI", s, e, s, e))
        else:
            raise ValueError(variant)
    return segs


def dense_counts(n: int, depth: int, variant: str) -> tuple[int, int]:
    """Tables 1-2 quantities for a DENSE triangle:
    b-updates = n (every triangle updates its own b once) + rows of every
    off-diagonal block; x-loads = columns of every off-diagonal block."""
    segs = partition(n, depth, variant)
    b_upd = n + sum(s.row1 - s.row0 for s in segs if s.kind == "SQ")
    x_ld = sum(s.col1 - s.col0 for s in segs if s.kind == "SQ")
    return b_upd, x_ld


# ---------------------------------------------------------------------------
# 6. Alg 7 decision tree (readings R8-R12)
# ---------------------------------------------------------------------------
def select_tri(nlevels: int, nnz_per_row: int) -> str:
    if nlevels == 1:
        return TRI_COMPLETELY_PARALLEL
    if nlevels > 20000:
        return TRI_NEAR_SERIAL
    if (nnz_per_row == 1 and nlevels <= 100) or (nnz_per_row <= 15 and nlevels <= 20):
        return TRI_LEVEL_SET
    return TRI_SYNC_FREE


def select_sq(nnz_per_row: int, empty_rows: int, nrows: int) -> str:
    # emptyratio = empty_rows / nrows, compared in integers (reading R9)
    if nnz_per_row <= 12 and 2 * empty_rows <= nrows:
        return SQ_SCALAR_CSR
    if nnz_per_row <= 12:
        return SQ_SCALAR_DCSR
    if 20 * empty_rows <= 3 * nrows:
        return SQ_VECTOR_CSR
    return SQ_VECTOR_DCSR


FORMAT_OF = {
    TRI_COMPLETELY_PARALLEL: "DIAG",
    TRI_LEVEL_SET: "CSR",
    TRI_SYNC_FREE: "CSR",
    TRI_NEAR_SERIAL: "CSR",
    SQ_SCALAR_CSR: "CSR",
    SQ_VECTOR_CSR: "CSR",
    SQ_SCALAR_DCSR: "DCSR",
    SQ_VECTOR_DCSR: "DCSR",
}


# ---------------------------------------------------------------------------
# 2 + 3 + 5: the full analysis
# ---------------------------------------------------------------------------
def _reverse(row_ptr, col_idx, n):
    """J U J for an upper CSR: row i -> n-1-i, col j -> n-1-j (reading R19)."""
    rp = row_ptr.astype(np.int64)
    rows = np.repeat(np.arange(n, dtype=np.int64), np.diff(rp))
    nr = n - 1 - rows
    nc = n - 1 - col_idx.astype(np.int64)
    order = np.lexsort((nc, nr))
    rp2 = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(nr, minlength=n), out=rp2[1:])
    return rp2, nc[order], order


@dataclasses.dataclass
class Analysis:
    n: int
    nnz: int
    depth: int
    variant: str
    perm: np.ndarray  # new -> old (original indices)
    leaf_level: np.ndarray  # level of each new row inside its leaf triangle
    segs: list
    seg_arrays: list  # per seg dict: IN_DEGREE / LEVEL_PTR / DCSR_ROWS
    # the final permuted lower-triangular matrix P L P^T (J U J for upper)
    p_row_ptr: np.ndarray = None
    p_col_idx: np.ndarray = None
    p_val: np.ndarray = None


def analyse(M, min_block_rows: int | None = None, depth: int | None = None,
            variant: str = "REC", reorder: bool = True) -> Analysis:
    """Run the paper's preprocessing on M (CSR, uplo "L" or "U")."""
    n = M.n
    rp = M.row_ptr.astype(np.int64)
    ci = M.col_idx.astype(np.int64)
    val = np.asarray(M.val)
    rev_order = None
    if M.uplo == "U":
        rp, ci, rev_order = _reverse(M.row_ptr, M.col_idx, n)
        val = val[rev_order]
    # off-diagonal entries of every original row (the diagonal is last)
    if depth is None:
        d = depth_rule(n, min_block_rows) if n else 0
    else:
        d = clamp_depth(n, depth)
    perm = np.arange(n, dtype=np.int64)  # new -> old
    old2new = np.arange(n, dtype=np.int64)
    leaf_level = np.zeros(n, dtype=np.int32)
    leaf_nlev = {}

    def sub_csr(lo, hi):
        """Off-diagonal entries of the current P L P^T restricted to
        rows/cols [lo, hi), local indices."""
        rows_old = perm[lo:hi]
        starts = rp[rows_old]
        lens = rp[rows_old + 1] - 1 - starts  # exclude the diagonal
        tot = int(lens.sum())
        loc_row = np.repeat(np.arange(hi - lo, dtype=np.int64), lens)
        offs = np.zeros(hi - lo + 1, dtype=np.int64)
        np.cumsum(lens, out=offs[1:])
        idx = starts[loc_row] + (np.arange(tot, dtype=np.int64) - offs[loc_row])
        cnew = old2new[ci[idx]]
        keep = (cnew >= lo) & (cnew < hi)
        loc_row = loc_row[keep]
        lrp = np.zeros(hi - lo + 1, dtype=np.int64)
        np.cumsum(np.bincount(loc_row, minlength=hi - lo), out=lrp[1:])
        return lrp, (cnew[keep] - lo).astype(np.int32)

    def reorder_node(lo, hi):
        lrp, lci = sub_csr(lo, hi)
        lev, nl = levels_sweep(hi - lo, lrp, lci)
        if reorder:
            p = np.argsort(lev, kind="stable")  # ties keep current order (R4)
            perm[lo:hi] = perm[lo:hi][p]
            old2new[perm[lo:hi]] = np.arange(lo, hi, dtype=np.int64)
            lev = lev[p]
        return lev, nl

    def node(lo, hi, dd):
        lev, nl = reorder_node(lo, hi)  # every node, root and leaves (R3)
        if dd == 0:
            leaf_level[lo:hi] = lev
            leaf_nlev[lo] = nl
            return
        mid = lo + (hi - lo) // 2
        node(lo, mid, dd - 1)
        node(mid, hi, dd - 1)

    if n:
        node(0, n, d)

    # final P L P^T with sorted columns (R6)
    counts = np.diff(rp)
    rows_old = np.repeat(np.arange(n, dtype=np.int64), counts)
    new_r = old2new[rows_old]
    new_c = old2new[ci]
    order = np.lexsort((new_c, new_r))
    p_rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(new_r, minlength=n), out=p_rp[1:])
    p_ci = new_c[order]
    p_val = val[order]
    p_rows = new_r[order]

    segs = partition(n, d, variant)
    seg_arrays = []
    for s in segs:
        m = s.row1 - s.row0
        sel_r = slice(p_rp[s.row0], p_rp[s.row1])
        r_loc = p_rows[sel_r] - s.row0
        c_blk = p_ci[sel_r]
        inb = (c_blk >= s.col0) & (c_blk < s.col1)
        per_row = np.bincount(r_loc[inb], minlength=m)
        s.nnz = int(per_row.sum())
        s.nnz_per_row = s.nnz // m if m else 0  # integer nnz/row (R8)
        arrays = {}
        if s.kind == "TRI":
            s.nlevels = leaf_nlev[s.row0]
            s.kernel = select_tri(s.nlevels, s.nnz_per_row)
            arrays["IN_DEGREE"] = (per_row - 1).astype(np.int32)  # off-diagonals (R15)
            lv = leaf_level[s.row0:s.row1]
            lp = np.zeros(s.nlevels + 1, dtype=np.int32)
            np.cumsum(np.bincount(lv, minlength=s.nlevels), out=lp[1:])
            arrays["LEVEL_PTR"] = lp
        else:
            s.empty_rows = int((per_row == 0).sum())
            s.kernel = select_sq(s.nnz_per_row, s.empty_rows, m)
            arrays["DCSR_ROWS"] = np.nonzero(per_row)[0].astype(np.int32)
        s.format = FORMAT_OF[s.kernel]
        seg_arrays.append(arrays)

    perm_orig = perm if M.uplo == "L" else (n - 1 - perm)
    return Analysis(n=n, nnz=int(rp[-1]) if n else 0, depth=d, variant=variant,
                    perm=perm_orig.astype(np.int32), leaf_level=leaf_level, segs=segs,
                    seg_arrays=seg_arrays, p_row_ptr=p_rp, p_col_idx=p_ci, p_val=p_val)
