"""Seeded generators for the five BASELINE.json configs and adversarial shapes.

Conventions:
  * RNG: numpy Generator(PCG64(seed)), seed = 20200817 + k for L, +1000 for b.
  * CSR, int32 indices, fp64 values, columns strictly ascending in every row,
    the diagonal is the LAST entry of its row (Alg 1).
  * Off-diagonal values l_ij = +-U[0.5,1) / (2 k_i), k_i = off-diagonal count
    of row i, so sum_j |l_ij| < 1/2; diagonal d_i = 1 + U[0,0.25).
    (C2 is the exception: exact IC(0) factor of the 5-point Laplacian.)
  * RHS b ~ U[-1,1) i.i.d., returned with numpy shape (nrhs, n) in C order,
    i.e. column-major n x nrhs with leading dimension n.

Nothing here solves, levels, reorders or blocks anything.
"""
from __future__ import annotations

import dataclasses
import os

import numpy as np

SEED_BASE = 20200817


@dataclasses.dataclass
class Matrix:
    """A sparse triangular matrix in CSR (0-based, int32 indices)."""

    n: int
    row_ptr: np.ndarray  # int32 [n+1]
    col_idx: np.ndarray  # int32 [nnz]
    val: np.ndarray  # float64 [nnz]
    name: str = ""
    meta: dict = dataclasses.field(default_factory=dict)
    uplo: str = "L"

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    def astype(self, dtype) -> "Matrix":
        return dataclasses.replace(self, val=self.val.astype(dtype))


def _rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def _assemble(n: int, rows: np.ndarray, cols: np.ndarray, rng: np.random.Generator,
              name: str, meta: dict | None = None) -> Matrix:
    """Build a lower-triangular CSR from strictly-lower (row, col) pairs.

    Duplicates are removed, every row gets a diagonal (last in the row), and
    values follow the module's value model.
    """
    rows = np.asarray(rows, dtype=np.int64)
    cols = np.asarray(cols, dtype=np.int64)
    assert np.all(cols < rows), "generator produced a non-strictly-lower entry"
    diag = np.arange(n, dtype=np.int64)
    key = np.concatenate([rows * n + cols, diag * n + diag])
    key = np.unique(key)  # sorted, de-duplicated; diagonal sorts last in its row
    r = (key // n).astype(np.int64)
    c = (key % n).astype(np.int32)
    del key
    counts = np.bincount(r, minlength=n)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    k = counts - 1  # off-diagonal count per row
    nnz = int(row_ptr[-1])
    val = np.empty(nnz, dtype=np.float64)
    is_diag = c.astype(np.int64) == r
    m_off = int(nnz - n)
    sign = np.where(rng.random(m_off) < 0.5, -1.0, 1.0)
    mag = 0.5 + 0.5 * rng.random(m_off)
    kk = k[r[~is_diag]]
    val[~is_diag] = sign * mag / (2.0 * kk)
    val[is_diag] = 1.0 + 0.25 * rng.random(n)
    if row_ptr[-1] >= 2**31:
        raise ValueError("nnz does not fit int32 row_ptr")
    return Matrix(n=n, row_ptr=row_ptr.astype(np.int32), col_idx=c, val=val,
                  name=name, meta=dict(meta or {}))


# ---------------------------------------------------------------------------
# C1: random lower triangle, n=1000, min(i,4) distinct off-diagonals per row
# ---------------------------------------------------------------------------
def c1_random(n: int = 1000, k_max: int = 4, seed: int = SEED_BASE + 1) -> Matrix:
    rng = _rng(seed)
    rows, cols = [], []
    for i in range(1, n):
        k = min(i, k_max)
        cs = rng.choice(i, size=k, replace=False)
        rows.append(np.full(k, i))
        cols.append(cs)
    rows = np.concatenate(rows) if rows else np.zeros(0, np.int64)
    cols = np.concatenate(cols) if cols else np.zeros(0, np.int64)
    return _assemble(n, rows, cols, rng, "C1", {"k_max": k_max})


# ---------------------------------------------------------------------------
# C2: IC(0) factor of the 2D 5-point Laplacian on an nx x ny grid (x fastest)
# ---------------------------------------------------------------------------
def c2_laplacian_ic0(nx: int = 1000, ny: int | None = None) -> Matrix:
    """Exact IC(0) factor of A = 5-point Laplacian (diag 4, neighbours -1).

    l_{i,i-1} = -1/d_{i-1} (ix>0), l_{i,i-nx} = -1/d_{i-nx} (iy>0),
    d_i = sqrt(4 - l_{i,i-1}^2 - l_{i,i-nx}^2).  Deterministic (no RNG).
    The recurrence is evaluated along anti-diagonals for speed (input
    construction, not the triangular solve).
    """
    ny = nx if ny is None else ny
    n = nx * ny
    d = np.zeros((ny, nx), dtype=np.float64)
    for s in range(nx + ny - 1):
        iy = np.arange(max(0, s - nx + 1), min(ny - 1, s) + 1)
        ix = s - iy
        acc = np.full(iy.shape, 4.0)
        m = ix > 0
        acc[m] -= (1.0 / d[iy[m], ix[m] - 1]) ** 2
        m = iy > 0
        acc[m] -= (1.0 / d[iy[m] - 1, ix[m]]) ** 2
        d[iy, ix] = np.sqrt(acc)
    dflat = d.reshape(-1)
    i = np.arange(n, dtype=np.int64)
    ix = i % nx
    iy = i // nx
    has_s = iy > 0
    has_w = ix > 0
    counts = 1 + has_s.astype(np.int64) + has_w.astype(np.int64)
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    nnz = int(row_ptr[-1])
    col = np.empty(nnz, dtype=np.int32)
    val = np.empty(nnz, dtype=np.float64)
    pos = row_ptr[:-1].copy()
    # south neighbour (i - nx) first: it has the smaller column index
    col[pos[has_s]] = (i[has_s] - nx).astype(np.int32)
    val[pos[has_s]] = -1.0 / dflat[i[has_s] - nx]
    pos[has_s] += 1
    col[pos[has_w]] = (i[has_w] - 1).astype(np.int32)
    val[pos[has_w]] = -1.0 / dflat[i[has_w] - 1]
    pos[has_w] += 1
    col[pos] = i.astype(np.int32)
    val[pos] = dflat
    return Matrix(n=n, row_ptr=row_ptr.astype(np.int32), col_idx=col, val=val,
                  name="C2", meta={"nx": nx, "ny": ny})


# ---------------------------------------------------------------------------
# C3: layered power-law DAG with exactly P levels (vas_stokes_4M-shaped)
# ---------------------------------------------------------------------------
def c3_powerlaw_layers(n: int = 4_000_000, P: int = 2815, x_m: float = 6.8,
                       alpha: float = 1.5, k_cap: int = 5000,
                       seed: int = SEED_BASE + 3) -> Matrix:
    """Rows are emitted level by level; row i of level l>0 draws its first
    dependency uniformly from level l-1 (so its level is exactly l) and
    k_i-1 more from all earlier rows: half uniform, half 'hub' draws
    floor(start_l * U^3) that create long columns.  k_i is a Pareto(alpha)
    tail min(k_cap, floor(x_m U^(-1/alpha)), #earlier rows)."""
    rng = _rng(seed)
    if P > n:
        raise ValueError("P > n")
    w = rng.lognormal(0.0, 1.2, size=P)
    w = np.maximum(1, np.floor(w / w.sum() * n)).astype(np.int64)
    n_one = int(round(0.05 * P))
    if n_one:
        w[rng.choice(P, size=n_one, replace=False)] = 1
    big = int(np.argmax(w))
    w[big] += n - int(w.sum())
    if w[big] < 1:
        raise ValueError("level widths do not fit n")
    start = np.zeros(P + 1, dtype=np.int64)
    np.cumsum(w, out=start[1:])
    lev = np.repeat(np.arange(P, dtype=np.int64), w)  # level of every row
    row_start = start[lev]  # rows in earlier levels
    u = rng.random(n)
    k = np.floor(x_m * np.power(1.0 - u, -1.0 / alpha)).astype(np.int64)
    k = np.minimum(np.minimum(k, k_cap), row_start)
    k = np.where(lev > 0, np.maximum(k, 1), 0)
    tot = int(k.sum())
    rows = np.repeat(np.arange(n, dtype=np.int64), k)
    first = np.zeros(tot, dtype=bool)
    offs = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(k, out=offs[1:])
    first[offs[:-1][k > 0]] = True
    rs = row_start[rows]
    cols = np.empty(tot, dtype=np.int64)
    # first dependency: uniform over level l-1
    fr = rows[first]
    l_prev = lev[fr] - 1
    cols[first] = start[l_prev] + np.floor(rng.random(fr.size) * w[l_prev]).astype(np.int64)
    rest = ~first
    m = int(rest.sum())
    hub = rng.random(m) < 0.5
    uu = rng.random(m)
    rs_rest = rs[rest]
    c_rest = np.where(hub, np.floor(rs_rest * uu ** 3), np.floor(rs_rest * uu)).astype(np.int64)
    cols[rest] = np.minimum(c_rest, rs_rest - 1)
    del rs, first, rest, c_rest, uu, hub
    return _assemble(n, rows, cols, rng, "C3",
                     {"P": P, "x_m": x_m, "alpha": alpha, "level_widths": w})


# ---------------------------------------------------------------------------
# C4: supernodal factor, width-w supernodes, random recursive elimination tree
# ---------------------------------------------------------------------------
def c4_supernodal(n: int = 500_000, width: int = 64, seed: int = SEED_BASE + 4) -> Matrix:
    """Dense lower-triangular diagonal block per supernode plus dense
    off-diagonal tiles at the block rows of the parent p(J) ~ U(J, S-1] and
    grandparent p(p(J)).  Rows in postorder (supernode index order)."""
    rng = _rng(seed)
    S = (n + width - 1) // width
    sstart = np.arange(S + 1, dtype=np.int64) * width
    sstart[-1] = n
    parent = np.full(S, -1, dtype=np.int64)
    J = np.arange(S - 1, dtype=np.int64)
    parent[: S - 1] = J + 1 + np.floor(rng.random(S - 1) * (S - 1 - J)).astype(np.int64)
    parent[: S - 1] = np.minimum(parent[: S - 1], S - 1)
    tiles_I = [parent[: S - 1]]
    tiles_J = [J]
    gp_ok = parent[: S - 1] < S - 1
    tiles_I.append(parent[parent[: S - 1][gp_ok]])
    tiles_J.append(J[gp_ok])
    TI = np.concatenate(tiles_I)
    TJ = np.concatenate(tiles_J)
    ar = np.arange(width, dtype=np.int64)
    rows_l, cols_l = [], []
    chunk = 4096
    for a in range(0, TI.size, chunk):
        ti, tj = TI[a:a + chunk], TJ[a:a + chunk]
        rr = sstart[ti][:, None, None] + ar[None, :, None]
        cc = sstart[tj][:, None, None] + ar[None, None, :]
        rr, cc = np.broadcast_arrays(rr, cc)
        ok = (rr < sstart[ti + 1][:, None, None]) & (cc < sstart[tj + 1][:, None, None])
        rows_l.append(rr[ok])
        cols_l.append(cc[ok])
    # strictly-lower part of each dense diagonal block
    ii, jj = np.tril_indices(width, -1)
    for a in range(0, S, chunk):
        s = np.arange(a, min(S, a + chunk), dtype=np.int64)
        rr = sstart[s][:, None] + ii[None, :]
        cc = sstart[s][:, None] + jj[None, :]
        ok = rr < sstart[s + 1][:, None]
        rows_l.append(rr[ok])
        cols_l.append(cc[ok])
    rows = np.concatenate(rows_l)
    cols = np.concatenate(cols_l)
    del rows_l, cols_l
    return _assemble(n, rows, cols, rng, "C4", {"width": width, "S": S, "parent": parent})


# ---------------------------------------------------------------------------
# C5: random, min(i,9) columns per row drawn with replacement (deduped)
# ---------------------------------------------------------------------------
def c5_random_multirhs(n: int = 2_000_000, k_max: int = 9, seed: int = SEED_BASE + 5) -> Matrix:
    rng = _rng(seed)
    i = np.arange(n, dtype=np.int64)
    k = np.minimum(i, k_max)
    rows = np.repeat(i, k)
    cols = np.floor(rng.random(rows.size) * rows).astype(np.int64)
    cols = np.minimum(cols, rows - 1)
    return _assemble(n, rows, cols, rng, "C5", {"k_max": k_max})


def gen_rhs(n: int, nrhs: int = 1, seed: int = SEED_BASE + 1000, dtype=np.float64) -> np.ndarray:
    """b ~ U[-1,1), numpy shape (nrhs, n) C-order == column-major n x nrhs."""
    rng = _rng(seed)
    return (2.0 * rng.random((nrhs, n)) - 1.0).astype(dtype)


def gen_rhs_cols(n: int, c0: int, c1: int, seed: int = SEED_BASE + 1000, dtype=np.float64) -> np.ndarray:
    """Columns [c0, c1) of gen_rhs(n, nrhs, seed) without drawing the others
    (PCG64 jump-ahead; one 64-bit draw per double), numpy shape (c1-c0, n).
    Lets every rank of a sharded SpTRSM create only its own shard."""
    bg = np.random.PCG64(seed)
    bg.advance(int(c0) * int(n))
    rng = np.random.Generator(bg)
    return (2.0 * rng.random((c1 - c0, n)) - 1.0).astype(dtype)


def config_seed(name: str) -> int:
    """Seed of a config's right-hand sides (gen_config)."""
    return SEED_BASE + int(name[1:]) + 1000


# name -> (builder, default nrhs); full BASELINE.json sizes
CONFIGS = {
    "C1": (lambda: c1_random(), 1),
    "C2": (lambda: c2_laplacian_ic0(), 1),
    "C3": (lambda: c3_powerlaw_layers(), 1),
    "C4": (lambda: c4_supernodal(), 1),
    "C5": (lambda: c5_random_multirhs(), 512),
}

# reduced sizes (same recipes) that the oracle finishes in seconds but that
# still span many tiles / CTAs and leave ragged tails
SMALL = {
    "C1": (lambda: c1_random(), 1),
    "C2": (lambda: c2_laplacian_ic0(nx=157, ny=131), 1),
    "C3": (lambda: c3_powerlaw_layers(n=60_013, P=97, x_m=6.8), 1),
    "C4": (lambda: c4_supernodal(n=20_011, width=64), 1),
    "C5": (lambda: c5_random_multirhs(n=50_021), 37),
}


def _build_cached(name: str, small: bool, build) -> Matrix:
    """build(), or its copy under $SPTRSV_GEN_CACHE (opt-in, for tuning
    scripts that regenerate the same full-size matrix many times)."""
    d = os.environ.get("SPTRSV_GEN_CACHE")
    if not d:
        return build()
    path = os.path.join(d, f"{name}{'_small' if small else ''}.npz")
    if os.path.exists(path):
        z = np.load(path)
        return Matrix(n=int(z["n"]), row_ptr=z["row_ptr"], col_idx=z["col_idx"], val=z["val"], name=str(z["name"]))
    L = build()
    os.makedirs(d, exist_ok=True)
    np.savez(path + ".tmp.npz", n=L.n, row_ptr=L.row_ptr, col_idx=L.col_idx, val=L.val, name=L.name)
    os.replace(path + ".tmp.npz", path)
    return L


def gen_config(name: str, small: bool = False, nrhs: int | None = None, dtype=np.float64):
    """Return (Matrix, b) for a config; b has numpy shape (nrhs, n)."""
    k = int(name[1:])
    build, default_nrhs = (SMALL if small else CONFIGS)[name]
    L = _build_cached(name, small, build)
    if dtype != np.float64:
        L = L.astype(dtype)
    nr = default_nrhs if nrhs is None else nrhs
    b = gen_rhs(L.n, nr, seed=config_seed(name), dtype=dtype)
    return L, b


def gen_matrix(name: str, small: bool = False, dtype=np.float64) -> Matrix:
    """The matrix of a config only (no right-hand side)."""
    L = (SMALL if small else CONFIGS)[name][0]()
    return L.astype(dtype) if dtype != np.float64 else L


# ---------------------------------------------------------------------------
# adversarial / special shapes
# ---------------------------------------------------------------------------
def shape_diagonal(n: int, seed: int = 7) -> Matrix:
    rng = _rng(seed)
    return _assemble(n, np.zeros(0), np.zeros(0), rng, "diagonal")


def shape_bidiagonal(n: int, a: float | None = None, seed: int = 8) -> Matrix:
    """Chain: row i depends on i-1 (n levels).  With a given, the sub-diagonal
    is -a and the diagonal 1 (closed-form inverse)."""
    rng = _rng(seed)
    i = np.arange(1, n)
    M = _assemble(n, i, i - 1, rng, "bidiagonal")
    if a is not None:
        off = np.ones(M.nnz, dtype=bool)
        off[M.row_ptr[1:] - 1] = False
        M.val[off] = -a
        M.val[~off] = 1.0
    return M


def shape_dense_lower(n: int, seed: int = 9) -> Matrix:
    rng = _rng(seed)
    r, c = np.tril_indices(n, -1)
    return _assemble(n, r, c, rng, "dense_lower")


def shape_arrow(n: int, seed: int = 10) -> Matrix:
    """Every row depends on row 0 (one long column) and the last row depends
    on everything (one long row)."""
    rng = _rng(seed)
    r1 = np.arange(1, n)
    c1 = np.zeros(n - 1, dtype=np.int64)
    r2 = np.full(max(n - 2, 0), n - 1)
    c2 = np.arange(1, n - 1)
    return _assemble(n, np.concatenate([r1, r2]), np.concatenate([c1, c2]), rng, "arrow")


def shape_paper_fig1() -> Matrix:
    """An 8x8 lower triangle with 15 nonzeros consistent with the text of
    PAPER.md:L73 (Fig. 1 itself is missing): x2, x3, x4 become solvable after
    x0, x1, x6; four level sets, the last two serial."""
    rng = _rng(11)
    off = [(2, 0), (3, 1), (4, 0), (4, 1), (5, 2), (5, 3), (7, 5)]
    r = np.array([a for a, _ in off])
    c = np.array([b for _, b in off])
    return _assemble(8, r, c, rng, "paper_fig1")


def shape_random_small(n: int, density: float, seed: int) -> Matrix:
    rng = _rng(seed)
    r, c = np.tril_indices(n, -1)
    keep = rng.random(r.size) < density
    return _assemble(n, r[keep], c[keep], rng, f"random_{n}_{density}")


def shape_long_rows(n: int = 6000, seed: int = 11) -> Matrix:
    """Rows of every length class of the row-block square kernel: empty,
    short (1-20), medium (257-1024 entries: one warp alone) and very long
    (> 1024: split into chunks), scattered over the lower half."""
    rng = _rng(seed)
    rows, cols = [], []
    for i in range(1, n):
        u = rng.random()
        if i < n // 2 or u < 0.2:
            k = min(i, int(rng.integers(0, 4)))
        elif u < 0.9:
            k = min(i, int(rng.integers(1, 21)))
        elif u < 0.97:
            k = min(i, int(rng.integers(257, 1025)))
        else:
            k = min(i, int(rng.integers(1025, 2900)))
        if k:
            c = rng.choice(i, size=k, replace=False)
            rows.append(np.full(k, i))
            cols.append(c)
    return _assemble(n, np.concatenate(rows), np.concatenate(cols), rng, "long_rows")


def to_upper(L: Matrix) -> Matrix:
    """U = J L J (index reversal i -> n-1-i): an upper-triangular CSR whose
    diagonal is the FIRST entry of its row.  Pure re-indexing."""
    n = L.n
    rows = np.repeat(np.arange(n, dtype=np.int64), np.diff(L.row_ptr.astype(np.int64)))
    nr = n - 1 - rows
    nc = n - 1 - L.col_idx.astype(np.int64)
    order = np.lexsort((nc, nr))
    counts = np.bincount(nr, minlength=n)
    rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    return Matrix(n=n, row_ptr=rp.astype(np.int32), col_idx=nc[order].astype(np.int32),
                  val=L.val[order].copy(), name=L.name + "_upper", meta=dict(L.meta), uplo="U")


def transpose(M: Matrix) -> Matrix:
    """M^T as CSR (the other fill): LOWER L -> upper L^T with the diagonal first
    in each row, UPPER U -> lower U^T with the diagonal last.  Pure re-indexing
    (a stable sort of the entries by (column, row)); the input of the
    transposed-solve parity tests (R31)."""
    n = M.n
    rows = np.repeat(np.arange(n, dtype=np.int64), np.diff(M.row_ptr.astype(np.int64)))
    cols = M.col_idx.astype(np.int64)
    order = np.lexsort((rows, cols))
    counts = np.bincount(cols, minlength=n)
    rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    return Matrix(n=n, row_ptr=rp.astype(np.int32), col_idx=rows[order].astype(np.int32),
                  val=M.val[order].copy(), name=M.name + "_T", meta=dict(M.meta),
                  uplo="U" if M.uplo == "L" else "L")
