// Host-side preprocessing of the recursive-block SpTRSV (the "analysis" of
// sptrsv_analyse).  Deterministic: the same input always gives the same plan,
// bit for bit, on any machine and thread count (needed for replicated plans
// across ranks).
//
// Steps, in the paper's order (see DESIGN.md sec. 3 for the numbered readings):
//   validate            Alg 1 layout: diagonal last in each CSR row
//   levels              Alg 2 (L77-L87): level(i) = 1 + max level of its dependencies
//   reorder             Sec 3.3 (L231-L233): stable sort of every triangle by level
//   recursive split     Alg 6 (L184-L195), mid = lo + floor(m/2); depth rule L299
//   COL / ROW variants  Alg 4 (L149-L159) / Alg 5 (L166-L176), same leaves (L182)
//   blocked storage     Sec 3.3 (L229, L235-L241): triangles and squares in
//                       execution order, diagonal separate, CSR or DCSR
//   features + Alg 7    Sec 3.4 (L252-L296)
#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <memory>
#include <mutex>
#include <numeric>
#include <thread>

#include "internal.h"

namespace sptrsv {

namespace {

// Run f(lo, hi) over [0, n) split into contiguous chunks on `threads` threads.
void parallel_for(int64_t n, int threads, const std::function<void(int64_t, int64_t)>& f) {
  if (threads <= 1 || n < 65536) {
    f(0, n);
    return;
  }
  std::vector<std::thread> th;
  for (int t = 0; t < threads; ++t) {
    int64_t a = n * t / threads, b = n * (t + 1) / threads;
    th.emplace_back([=, &f] { f(a, b); });
  }
  for (auto& x : th) x.join();
}

// The lower-triangular input the analysis works on.  LOWER input is read in
// place (the caller's CSR outlives the blocking sptrsv_analyse call); UPPER
// is materialised as J U J.
struct LowerCSR {
  int32_t n = 0;
  std::vector<int64_t> rp;
  const int32_t* ci = nullptr;
  const char* val = nullptr;
  dvec<int32_t> ci_own;
  dvec<char> val_own;
};

// Row-local checks of one CSR row (the first failing check wins).
Error validate_row(int32_t i, int64_t nnz, int32_t n, const int32_t* rp, const int32_t* ci, const char* val,
                   size_t vb, sptrsv_fill_t fill) {
  int64_t s = rp[i], e = rp[i + 1];
  if (e < s || e > nnz) return {SPTRSV_ERROR_INVALID_VALUE, "row_ptr not monotone at row " + std::to_string(i)};
  for (int64_t q = s; q < e; ++q) {
    int32_t c = ci[q];
    if (c < 0 || c >= n) return {SPTRSV_ERROR_INVALID_VALUE, "column index out of range in row " + std::to_string(i)};
    if (q > s && c <= ci[q - 1]) return {SPTRSV_ERROR_UNSORTED, "columns not strictly increasing in row " + std::to_string(i)};
  }
  bool zero;
  if (fill == SPTRSV_LOWER) {
    if (e > s && ci[e - 1] > i) return {SPTRSV_ERROR_NOT_TRIANGULAR, "entry above the diagonal in row " + std::to_string(i)};
    if (e == s || ci[e - 1] != i) return {SPTRSV_ERROR_ZERO_PIVOT, "missing diagonal in row " + std::to_string(i)};
    const char* d = val + (size_t)(e - 1) * vb;
    zero = vb == 8 ? (*(const double*)d == 0.0) : (*(const float*)d == 0.0f);
  } else {
    if (e > s && ci[s] < i) return {SPTRSV_ERROR_NOT_TRIANGULAR, "entry below the diagonal in row " + std::to_string(i)};
    if (e == s || ci[s] != i) return {SPTRSV_ERROR_ZERO_PIVOT, "missing diagonal in row " + std::to_string(i)};
    const char* d = val + (size_t)s * vb;
    zero = vb == 8 ? (*(const double*)d == 0.0) : (*(const float*)d == 0.0f);
  }
  if (zero) return {SPTRSV_ERROR_ZERO_PIVOT, "zero diagonal in row " + std::to_string(i)};
  return {SPTRSV_SUCCESS, ""};
}

// Rows are checked in parallel chunks; the error reported is the one of the
// lowest failing row, exactly what a serial row-order scan reports.
Error validate(int32_t n, int64_t nnz, const int32_t* rp, const int32_t* ci, const char* val, size_t vb,
               sptrsv_fill_t fill, int threads) {
  if (rp[0] != 0) return {SPTRSV_ERROR_INVALID_VALUE, "row_ptr[0] != 0"};
  if ((int64_t)rp[n] != nnz) return {SPTRSV_ERROR_INVALID_VALUE, "nnz != row_ptr[n]"};
  // a monotone row_ptr is checked first (n reads) so every chunk may index
  // its rows safely; a violation is reported by a serial scan up to it
  for (int32_t i = 0; i < n; ++i)
    if (rp[i + 1] < rp[i] || rp[i + 1] > nnz) {
      for (int32_t j = 0; j <= i; ++j) {
        Error e = validate_row(j, nnz, n, rp, ci, val, vb, fill);
        if (e.status) return e;
      }
    }
  std::mutex mu;
  int32_t best = -1;
  Error best_e{SPTRSV_SUCCESS, ""};
  parallel_for(n, threads, [&](int64_t a, int64_t b) {
    for (int64_t i = a; i < b; ++i) {
      Error e = validate_row((int32_t)i, nnz, n, rp, ci, val, vb, fill);
      if (e.status) {
        std::lock_guard<std::mutex> g(mu);
        if (best < 0 || i < best) {
          best = (int32_t)i;
          best_e = e;
        }
        return;
      }
    }
  });
  return best_e;
}

// Lower CSR of the input; UPPER is mapped to J U J (i -> n-1-i, reading R19):
// row n-1-i of the result is row i of U read backwards, so its columns are
// ascending and the diagonal (first in U's row) becomes last.
void to_lower(LowerCSR& L, int32_t n, const int32_t* rp, const int32_t* ci, const char* val, size_t vb,
              sptrsv_fill_t fill, int threads) {
  L.n = n;
  int64_t nnz = rp[n];
  L.rp.resize((size_t)n + 1);
  if (fill == SPTRSV_LOWER) {
    for (int32_t i = 0; i <= n; ++i) L.rp[i] = rp[i];
    L.ci = ci;
    L.val = val;
    return;
  }
  L.ci_own.resize((size_t)nnz);
  L.val_own.resize((size_t)nnz * vb);
  L.rp[0] = 0;
  for (int32_t r = 0; r < n; ++r) {
    int32_t i = n - 1 - r;
    L.rp[r + 1] = L.rp[r] + (rp[i + 1] - rp[i]);
  }
  parallel_for(n, threads, [&](int64_t a, int64_t b) {
    for (int64_t r = a; r < b; ++r) {
      int32_t i = n - 1 - (int32_t)r;
      int64_t o = L.rp[r];
      for (int64_t q = (int64_t)rp[i + 1] - 1; q >= rp[i]; --q, ++o) {
        L.ci_own[o] = n - 1 - ci[q];
        std::memcpy(&L.val_own[(size_t)o * vb], val + (size_t)q * vb, vb);
      }
    }
  });
  L.ci = L.ci_own.data();
  L.val = L.val_own.data();
}

// Lower CSR of the transposed input (R31): the
// plan then solves A^T x = b.  A = L (LOWER): L^T is upper and is mapped to
// J L^T J, entry (i, j) -> (n-1-j, n-1-i); A = U (UPPER): U^T is lower as is,
// entry (i, j) -> (j, i).  A counting sort by destination row; source rows are
// walked in the order that makes every destination row's columns ascending
// (descending i for L, ascending i for U), so the diagonal lands last.
void to_lower_transposed(LowerCSR& L, int32_t n, const int32_t* rp, const int32_t* ci, const char* val,
                         size_t vb, sptrsv_fill_t fill) {
  L.n = n;
  int64_t nnz = rp[n];
  const bool low = fill == SPTRSV_LOWER;
  L.rp.assign((size_t)n + 1, 0);
  for (int64_t q = 0; q < nnz; ++q) {
    int32_t r = low ? n - 1 - ci[q] : ci[q];
    ++L.rp[(size_t)r + 1];
  }
  for (int32_t r = 0; r < n; ++r) L.rp[r + 1] += L.rp[r];
  std::vector<int64_t> pos(L.rp.begin(), L.rp.end() - 1);
  L.ci_own.resize((size_t)nnz);
  L.val_own.resize((size_t)nnz * vb);
  for (int32_t t = 0; t < n; ++t) {
    int32_t i = low ? n - 1 - t : t;
    int32_t c = low ? n - 1 - i : i;
    for (int64_t q = rp[i]; q < rp[i + 1]; ++q) {
      int32_t r = low ? n - 1 - ci[q] : ci[q];
      int64_t o = pos[r]++;
      L.ci_own[o] = c;
      std::memcpy(&L.val_own[(size_t)o * vb], val + (size_t)q * vb, vb);
    }
  }
  L.ci = L.ci_own.data();
  L.val = L.val_own.data();
}

// Reading R2: largest d with d == 0 or floor(n / 2^d) >= T.
// The depth-rule threshold T of L299 ("20 x CUDA cores"; reading R2).
// Under the B200 selector with neither depth nor min_block_rows given, T is
// 4x the paper's (reading R33): re-derived on B200 by the depth sweep of
// DESIGN.md 5.8 (C3 depth 3 -> 1: -2.5%; C5 2 -> 0: -11% at 512 RHS, -13%
// at one RHS; C1 / C2 / C4 unchanged), the L299 experiment redone on this
// GPU with its kernels.  SPTRSV_NO_DEPTH_RETUNE keeps the paper's T.
int64_t min_block_rows_rule(const Plan& p) {
  if (p.opts.min_block_rows > 0) return p.opts.min_block_rows;
  const int64_t T = (int64_t)20 * p.sm_count * 128;
  if (p.opts.selector == SPTRSV_SELECT_B200 && p.opts.depth < 0 && std::getenv("SPTRSV_NO_DEPTH_RETUNE") == nullptr)
    return 4 * T;
  return T;
}

int32_t depth_rule(int64_t n, int64_t T) {
  int32_t d = 0;
  while ((n >> (d + 1)) >= T) ++d;
  return d;
}

// Reading R1b: a forced depth keeps at least one row per leaf.
int32_t clamp_depth(int64_t n, int32_t d) {
  if (n <= 1) return 0;
  int32_t lg = 0;
  while ((int64_t(1) << (lg + 1)) <= n) ++lg;
  return std::min(d, lg);
}

// Fundamental supernodes, cut into pieces of <= kSnMax rows: row r joins the
// piece of row r-1 iff its off-diagonal columns are exactly those of row
// r-1 plus r-1 itself (so the piece's diagonal block is dense and its rows
// share one list of external columns).  Returns the number of pieces.
constexpr int32_t kSnMax = 32;

int64_t supernode_pieces(int32_t n, const std::vector<int64_t>& rp, const int32_t* ci,
                         std::vector<int32_t>* starts) {
  int64_t np = 0;
  int32_t start = 0;
  for (int32_t r = 0; r < n; ++r) {
    bool join = false;
    if (r > start && r - start < kSnMax) {
      const int64_t a0 = rp[r - 1], l0 = rp[r] - 1 - a0;  // off-diagonals of r-1
      const int64_t a1 = rp[r], l1 = rp[r + 1] - 1 - a1;  // off-diagonals of r
      join = l1 == l0 + 1 && ci[a1 + l1 - 1] == r - 1 &&
             std::equal(ci + a0, ci + a0 + l0, ci + a1);
    }
    if (!join) {
      start = r;
      ++np;
      if (starts) starts->push_back(r);
    }
  }
  if (starts) starts->push_back(n);
  return np;
}

struct Reorderer {
  const LowerCSR& L;
  bool reorder;
  std::vector<int32_t> perm, old2new, leaf_level;

  explicit Reorderer(const LowerCSR& l, bool re) : L(l), reorder(re) {
    perm.resize(L.n);
    old2new.resize(L.n);
    leaf_level.assign(L.n, 0);
    std::iota(perm.begin(), perm.end(), 0);
    std::iota(old2new.begin(), old2new.end(), 0);
  }

  // Levels of the triangle rows/cols [lo,hi) of the current P L P^T (only
  // dependencies inside the triangle count, reading R5), then a stable
  // counting sort of its rows by level (ties keep the current order, R4).
  // Writes the (sorted) levels into leaf_level[lo,hi); returns nlevels.
  // Levels of rows [lo, hi) by threads working on consecutive row chunks
  // in claim order: a dependency in an earlier chunk that is still being
  // swept is waited for (its level slot holds -1 until written), and the
  // lowest unfinished chunk never waits, so the sweep cannot deadlock.  The
  // levels are the serial sweep's exactly (each is 1 + the max over its
  // dependencies, however the work is split).
  int32_t levels_parallel(int32_t lo, int32_t hi, bool identity, int threads, std::vector<int32_t>& lev) {
    const int32_t m = hi - lo;
    constexpr int32_t CH = 2048;
    const int32_t nch = (m + CH - 1) / CH;
    std::unique_ptr<std::atomic<int32_t>[]> al(new std::atomic<int32_t>[(size_t)m]);
    par_for(m, threads, [&](int64_t a, int64_t b) {
      for (int64_t k = a; k < b; ++k) al[k].store(-1, std::memory_order_relaxed);
    });
    std::atomic<int32_t> next{0};
    std::vector<int32_t> tmax((size_t)threads, 0);
    std::vector<std::thread> th;
    for (int t = 0; t < threads; ++t)
      th.emplace_back([&, t] {
        int32_t mx = 0;
        for (int32_t ch; (ch = next.fetch_add(1, std::memory_order_relaxed)) < nch;) {
          const int32_t r1 = lo + std::min(m, (ch + 1) * CH);
          for (int32_t r = lo + ch * CH; r < r1; ++r) {
            const int32_t o = identity ? r : perm[r];
            int32_t lv = 0;
            for (int64_t q = L.rp[o], e = L.rp[o + 1] - 1; q < e; ++q) {
              const int32_t c = identity ? L.ci[q] : old2new[L.ci[q]];
              if (c < lo) continue;
              int32_t v = al[c - lo].load(std::memory_order_acquire);
              while (v < 0) {
#if defined(__x86_64__) || defined(__i386__)
                __builtin_ia32_pause();
#endif
                v = al[c - lo].load(std::memory_order_acquire);
              }
              lv = std::max(lv, v + 1);
            }
            al[r - lo].store(lv, std::memory_order_release);
            mx = std::max(mx, lv + 1);
          }
        }
        tmax[t] = mx;
      });
    for (auto& x : th) x.join();
    par_for(m, threads, [&](int64_t a, int64_t b) {
      for (int64_t k = a; k < b; ++k) lev[k] = al[k].load(std::memory_order_relaxed);
    });
    return *std::max_element(tmax.begin(), tmax.end());
  }

  int32_t node_reorder(int32_t lo, int32_t hi, bool identity = false, int inner = 1) {
    int32_t m = hi - lo;
    if (m == 0) return 0;
    std::vector<int32_t> lev((size_t)m);
    int32_t nl = 0;
    if (inner > 1 && m >= 65536) {
      nl = levels_parallel(lo, hi, identity, inner, lev);
    } else if (identity) {  // perm is still the identity (the root): no old2new lookups
      for (int32_t r = lo; r < hi; ++r) {
        int32_t lv = 0;
        for (int64_t q = L.rp[r], e = L.rp[r + 1] - 1; q < e; ++q) {
          int32_t c = L.ci[q];
          if (c >= lo) lv = std::max(lv, lev[c - lo] + 1);
        }
        lev[r - lo] = lv;
        nl = std::max(nl, lv + 1);
      }
    } else {
      for (int32_t r = lo; r < hi; ++r) {
        int32_t o = perm[r];
        int32_t lv = 0;
        for (int64_t q = L.rp[o], e = L.rp[o + 1] - 1; q < e; ++q) {  // off-diagonals
          int32_t c = old2new[L.ci[q]];
          if (c >= lo) lv = std::max(lv, lev[c - lo] + 1);
        }
        lev[r - lo] = lv;
        nl = std::max(nl, lv + 1);
      }
    }
    if (reorder) {
      std::vector<int32_t> cnt((size_t)nl + 1, 0);
      for (int32_t k = 0; k < m; ++k) cnt[lev[k] + 1]++;
      for (int32_t l = 0; l < nl; ++l) cnt[l + 1] += cnt[l];
      std::vector<int32_t> np((size_t)m);
      for (int32_t k = 0; k < m; ++k) np[cnt[lev[k]]++] = perm[lo + k];
      for (int32_t k = 0; k < m; ++k) {
        perm[lo + k] = np[k];
        old2new[np[k]] = lo + k;
      }
      // the sorted levels straight from the counts (cnt[l] is now the end of
      // level l's range)
      for (int32_t l = 0, k = 0; l < nl; ++l)
        for (; k < cnt[l]; ++k) lev[k] = l;
    }
    std::copy(lev.begin(), lev.end(), leaf_level.begin() + lo);
    return nl;
  }
};

}  // namespace

int32_t select_tri(int32_t nlevels, int32_t npr) {
  // Alg 7, PAPER.md:L270-L278 (branch order: reading R12)
  if (nlevels == 1) return SPTRSV_K_COMPLETELY_PARALLEL;
  if (nlevels > 20000) return SPTRSV_K_NEAR_SERIAL;
  if ((npr == 1 && nlevels <= 100) || (npr <= 15 && nlevels <= 20)) return SPTRSV_K_LEVEL_SET;
  return SPTRSV_K_SYNC_FREE;
}

int32_t select_sq(int32_t npr, int64_t empty, int64_t m) {
  // Alg 7, PAPER.md:L281-L292 with L258's thresholds; emptyratio compared in
  // integers (reading R9)
  if (npr <= 12) return (2 * empty <= m) ? SPTRSV_K_SCALAR_CSR : SPTRSV_K_SCALAR_DCSR;
  return (20 * empty <= 3 * m) ? SPTRSV_K_VECTOR_CSR : SPTRSV_K_VECTOR_DCSR;
}

Error analyse_host(Plan& p, int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx,
                   const void* val_v) {
  const char* val = (const char*)val_v;
  const size_t vb = p.vbytes;
  int threads = p.opts.threads > 0 ? p.opts.threads : (int)std::max(1u, std::thread::hardware_concurrency());
  threads = std::min(threads, 64);

  PhaseClock clk;
  Error e = validate(n, nnz, row_ptr, col_idx, val, vb, p.fill, threads);
  if (e.status) return e;
  clk.lap("validate");
  LowerCSR L;
  if (p.opts.transpose) {
    // the system solved is A^T: its fill is the other one (R31)
    to_lower_transposed(L, n, row_ptr, col_idx, val, vb, p.fill);
    p.fill = p.fill == SPTRSV_LOWER ? SPTRSV_UPPER : SPTRSV_LOWER;
  } else {
    to_lower(L, n, row_ptr, col_idx, val, vb, p.fill, threads);
  }
  clk.lap("to_lower");
  p.n = n;
  p.nnz = nnz;

  // ---- depth (L299) ----
  p.min_block_rows = min_block_rows_rule(p);
  if (p.opts.depth >= 0)
    p.depth = clamp_depth(n, p.opts.depth);
  else
    p.depth = n ? depth_rule(n, p.min_block_rows) : 0;
  // reading R33: the B200 threshold is 4x the paper's; report when it chose
  // a shallower tree than the paper's T would have
  if (p.opts.depth < 0 && n && p.min_block_rows != (int64_t)20 * p.sm_count * 128 && p.opts.min_block_rows == 0 &&
      p.depth < depth_rule(n, (int64_t)20 * p.sm_count * 128))
    p.depth_retuned = 3;

  // ---- recursive reordering: every node, root and leaves (reading R3) ----
  // Siblings are independent once their parent is reordered (each only reads
  // dependencies inside its own range), so one depth level runs in parallel.
  // reorder AUTO (reading R29): a supernodal input keeps its order, because
  // level sorting scatters the rows of every dense diagonal block over as
  // many levels as the block is wide (SURVEY.md 7.3 hard part 5)
  p.reorder_eff = p.opts.reorder == 1 ? 1 : 0;
  if (p.opts.reorder == 2 && n > 0) {
    const int64_t np = supernode_pieces(n, L.rp, L.ci, nullptr);
    p.reorder_eff = (np > 0 && (double)n / (double)np >= 8.0) ? 1 : 0;
  }
  Reorderer R(L, p.reorder_eff == 0);
  std::vector<int32_t> leaf_nl;
  std::vector<std::pair<int32_t, int32_t>> nodes = {{0, n}};
  for (int32_t d = 0; d <= p.depth && n > 0; ++d) {
    std::vector<int32_t> nl(nodes.size());
    // A top child [lo, mid) needs no work: its rows depend only on rows
    // < mid, so their levels inside [lo, mid) are the parent's (already in
    // leaf_level, and already sorted when reordering) and its stable level
    // sort is the identity (reading R3's invariant).  Only bottom children
    // (and the root) are analysed, in parallel.
    std::vector<size_t> work;
    for (size_t k = 0; k < nodes.size(); ++k) {
      if (d > 0 && k % 2 == 0) {
        int32_t mx = -1;
        for (int32_t r = nodes[k].first; r < nodes[k].second; ++r) mx = std::max(mx, R.leaf_level[r]);
        nl[k] = mx + 1;
      } else {
        work.push_back(k);
      }
    }
    if (work.size() == 1 || threads == 1) {
      // a lone node (the root, the first bottom child): swept by all threads
      // (measured: on C3's layered DAG two or more bottom nodes go faster
      // one thread each than one after the other swept in parallel)
      for (size_t k : work) nl[k] = R.node_reorder(nodes[k].first, nodes[k].second, d == 0, threads);
    } else {
      std::vector<std::thread> th;
      int T = std::min<int>(threads, (int)work.size());
      for (int t = 0; t < T; ++t)
        th.emplace_back([&, t] {
          for (size_t w = t; w < work.size(); w += T) nl[work[w]] = R.node_reorder(nodes[work[w]].first, nodes[work[w]].second);
        });
      for (auto& x : th) x.join();
    }
    if (clk.on) clk.lap(("  reorder depth " + std::to_string(d)).c_str());
    // Depth retune under the B200 selector (reading R30): a
    // root triangle whose levels are all narrow (<= 2048 rows) and whose rows
    // have 1..8 dependencies is solved whole by the strand wavefront, which
    // pipelines the level chain across the cluster; the paper's split
    // (L299) would only add a square and drain and refill the wavefront at
    // the kernel boundary (C2: 0.260 -> 0.215 ms).  Only when the caller left
    // both depth and min_block_rows to the library and level reordering is on.
    if (d == 0 && p.depth > 0 && p.opts.depth < 0 && p.opts.min_block_rows == 0 &&
        p.opts.selector == SPTRSV_SELECT_B200 && p.reorder_eff == 0 && n >= 4096 &&
        std::getenv("SPTRSV_NO_DEPTH_RETUNE") == nullptr) {
      std::vector<int32_t> wid((size_t)nl[0] + 1, 0);
      int32_t wmax = 0;
      for (int32_t r = 0; r < n; ++r) wmax = std::max(wmax, ++wid[R.leaf_level[r]]);
      int64_t kmin = INT64_MAX, kmax = 0;
      for (int32_t r = 0; r < n; ++r) {
        const int64_t k = L.rp[r + 1] - L.rp[r] - 1;
        kmin = std::min(kmin, k);
        kmax = std::max(kmax, k);
      }
      if (wmax <= 2048 && kmax >= 1 && kmax <= 8) {
        p.depth = 0;
        p.depth_retuned = 1;
      }
    }
    if (d == p.depth) {
      leaf_nl = nl;
      break;
    }
    std::vector<std::pair<int32_t, int32_t>> next;
    for (auto& nd : nodes) {
      int32_t mid = nd.first + (nd.second - nd.first) / 2;  // reading R1
      next.push_back({nd.first, mid});
      next.push_back({mid, nd.second});
    }
    nodes.swap(next);
  }

  clk.lap("levels + reorder");
  // ---- final P L P^T, columns sorted (reading R6) ----
  p.p_rp.assign((size_t)n + 1, 0);
  for (int32_t r = 0; r < n; ++r) {
    int32_t o = R.perm[r];
    p.p_rp[r + 1] = p.p_rp[r] + (L.rp[o + 1] - L.rp[o]);
  }
  p.p_ci.resize((size_t)nnz);
  p.p_val.resize((size_t)nnz * vb);
  parallel_for(n, threads, [&](int64_t a, int64_t b) {
    std::vector<std::pair<int32_t, int64_t>> tmp;
    for (int64_t r = a; r < b; ++r) {
      int32_t o = R.perm[r];
      int64_t s = L.rp[o], len = L.rp[o + 1] - s;
      int64_t d0 = p.p_rp[r];
      // map the columns; rows whose mapped columns stay ascending (all of
      // them without reordering, most of them with it) need no sort
      bool sorted = true;
      int32_t prev = -1;
      for (int64_t k = 0; k < len; ++k) {
        const int32_t c = R.old2new[L.ci[s + k]];
        p.p_ci[d0 + k] = c;
        sorted &= c > prev;
        prev = c;
      }
      if (sorted) {
        std::memcpy(&p.p_val[(size_t)d0 * vb], L.val + (size_t)s * vb, (size_t)len * vb);
        continue;
      }
      tmp.resize((size_t)len);
      for (int64_t k = 0; k < len; ++k) tmp[k] = {p.p_ci[d0 + k], s + k};
      std::sort(tmp.begin(), tmp.end());
      for (int64_t k = 0; k < len; ++k) {
        p.p_ci[d0 + k] = tmp[k].first;
        std::memcpy(&p.p_val[(size_t)(d0 + k) * vb], L.val + (size_t)tmp[k].second * vb, vb);
      }
    }
  });
  p.diag_new.resize((size_t)n * vb);
  p.rdiag_new.resize((size_t)n * vb);
  for (int32_t r = 0; r < n; ++r) {
    std::memcpy(&p.diag_new[(size_t)r * vb], &p.p_val[(size_t)(p.p_rp[r + 1] - 1) * vb], vb);
    if (vb == 8) {
      double v = 1.0 / *(const double*)&p.diag_new[(size_t)r * 8];
      std::memcpy(&p.rdiag_new[(size_t)r * 8], &v, 8);
    } else {
      float v = (float)(1.0 / (double)*(const float*)&p.diag_new[(size_t)r * 4]);
      std::memcpy(&p.rdiag_new[(size_t)r * 4], &v, 4);
    }
  }

  p.perm.resize(n);
  for (int32_t k = 0; k < n; ++k) p.perm[k] = p.fill == SPTRSV_LOWER ? R.perm[k] : n - 1 - R.perm[k];
  p.leaf_level = R.leaf_level;
  p.lower_old = R.perm;

  clk.lap("P L P^T");
  e = build_segments_host(p, nodes, leaf_nl, threads);
  if (e.status) return e;
  clk.lap("segments + Alg 7");
  choose_impls(p);
  clk.lap("choose_impls");
  return {SPTRSV_SUCCESS, ""};
}

// Segment geometry in execution order (Alg 4-6, readings R16-R18).
std::vector<SegGeo> segment_geometry(int32_t n, int32_t depth, int32_t variant,
                                     const std::vector<std::pair<int32_t, int32_t>>& leaves) {
  std::vector<SegGeo> geo;
  if (n > 0) {
    if (variant == SPTRSV_VARIANT_REC) {
      std::function<void(int32_t, int32_t, int32_t)> rec = [&](int32_t lo, int32_t hi, int32_t d) {
        if (d == 0) {
          int32_t li = (int32_t)(std::lower_bound(leaves.begin(), leaves.end(), std::make_pair(lo, hi)) - leaves.begin());
          geo.push_back({0, lo, hi, lo, hi, li});
          return;
        }
        int32_t mid = lo + (hi - lo) / 2;
        rec(lo, mid, d - 1);
        geo.push_back({1, mid, hi, lo, mid, -1});
        rec(mid, hi, d - 1);
      };
      rec(0, n, depth);
    } else {
      int32_t K = (int32_t)leaves.size();
      for (int32_t k = 0; k < K; ++k) {
        int32_t s = leaves[k].first, e2 = leaves[k].second;
        if (variant == SPTRSV_VARIANT_COL) {  // Alg 4, reading R16
          geo.push_back({0, s, e2, s, e2, k});
          if (k != K - 1) geo.push_back({1, e2, n, s, e2, -1});
        } else {  // Alg 5, reading R17
          if (k != 0) geo.push_back({1, s, e2, 0, s, -1});
          geo.push_back({0, s, e2, s, e2, k});
        }
      }
    }
  }
  return geo;
}

// Blocks, features and Alg 7 labels from the host P L P^T (p.p_rp / p_ci /
// p_val, p.diag_new, p.leaf_level); leaves = the recursion's leaf ranges in
// order, leaf_nl = their level counts.
Error build_segments_host(Plan& p, const std::vector<std::pair<int32_t, int32_t>>& nodes,
                          const std::vector<int32_t>& leaf_nl, int threads) {
  const int32_t n = p.n;
  const size_t vb = p.vbytes;
  // ---- segment geometry in execution order ----
  const std::vector<SegGeo> geo = segment_geometry(n, p.depth, p.opts.variant, nodes);

  // ---- extract blocks, features, Alg 7 ----
  p.segs.resize(geo.size());
  auto build_seg = [&](size_t si, int inner) {
    const SegGeo& g = geo[si];
    Segment& S = p.segs[si];
    sptrsv_seg_info_t& I = S.info;
    I.kind = g.kind;
    I.row0 = g.r0; I.row1 = g.r1; I.col0 = g.c0; I.col1 = g.c1;
    int32_t m = g.r1 - g.r0;
    S.rp.assign((size_t)m + 1, 0);
    dvec<int64_t> lo_idx((size_t)m), hi_idx((size_t)m);
    parallel_for(m, inner, [&](int64_t ka, int64_t kb) {
      for (int64_t k = ka; k < kb; ++k) {
        int32_t r = g.r0 + (int32_t)k;
        const int32_t* rb = p.p_ci.data() + p.p_rp[r];
        const int32_t* re = p.p_ci.data() + p.p_rp[r + 1];
        int32_t cend = g.kind == 0 ? r : g.c1;  // TRI: off-diagonals only
        const int32_t* a = std::lower_bound(rb, re, g.c0);
        const int32_t* b = std::lower_bound(a, re, cend);
        lo_idx[k] = a - p.p_ci.data();
        hi_idx[k] = b - p.p_ci.data();
      }
    });
    int64_t tot = 0, empty = 0;
    for (int32_t k = 0; k < m; ++k) {
      int64_t c = hi_idx[k] - lo_idx[k];
      tot += c;
      empty += (c == 0);
    }
    if (g.kind == 0) {
      I.nnz = tot + m;  // the diagonal counts (reading R8)
      I.nnz_per_row = m ? (int32_t)(I.nnz / m) : 0;
      I.nlevels = leaf_nl[g.leaf];
      I.empty_rows = 0;
      I.kernel = select_tri(I.nlevels, I.nnz_per_row);
      I.format = I.kernel == SPTRSV_K_COMPLETELY_PARALLEL ? SPTRSV_FMT_DIAG : SPTRSV_FMT_CSR;
      S.in_degree.resize(m);
      for (int32_t k = 0; k < m; ++k) S.in_degree[k] = (int32_t)(hi_idx[k] - lo_idx[k]);
      S.level_ptr.assign((size_t)I.nlevels + 1, 0);
      for (int32_t k = 0; k < m; ++k) S.level_ptr[p.leaf_level[g.r0 + k] + 1]++;
      int32_t mx = 0;
      for (int32_t l = 0; l < I.nlevels; ++l) {
        mx = std::max(mx, S.level_ptr[l + 1]);
        S.level_ptr[l + 1] += S.level_ptr[l];
      }
      I.max_level_rows = mx;
      S.nzr = m;
      {  // fundamental-supernode pieces of the triangle (its own entries only)
        S.sn_ptr.clear();
        // whether row k may extend row k-1's piece depends on those two rows
        // only (parallel); the 32-row cut is a serial pass
        std::vector<char> canj((size_t)m, 0);
        parallel_for(m, inner, [&](int64_t ka, int64_t kb) {
          for (int64_t k = std::max<int64_t>(ka, 1); k < kb; ++k) {
            const int64_t a0 = lo_idx[k - 1], l0 = hi_idx[k - 1] - a0;
            const int64_t a1 = lo_idx[k], l1 = hi_idx[k] - a1;
            canj[k] = l1 == l0 + 1 && p.p_ci[a1 + l1 - 1] == g.r0 + k - 1 &&
                      std::equal(p.p_ci.begin() + a0, p.p_ci.begin() + a0 + l0, p.p_ci.begin() + a1);
          }
        });
        int32_t start = 0;
        for (int32_t k = 0; k < m; ++k) {
          const bool join = k > start && k - start < kSnMax && canj[k];
          if (!join) {
            start = k;
            S.sn_ptr.push_back(k);
          }
        }
        S.sn_ptr.push_back(m);
      }
      S.npieces = (int64_t)S.sn_ptr.size() - 1;
      S.kmax_indeg = 0;
      for (int32_t k = 0; k < m; ++k) S.kmax_indeg = std::max(S.kmax_indeg, S.in_degree[k]);
    } else {
      I.nnz = tot;
      I.nnz_per_row = m ? (int32_t)(tot / m) : 0;
      I.empty_rows = (int32_t)empty;
      I.nlevels = 0;
      I.kernel = select_sq(I.nnz_per_row, empty, m);
      I.format = (I.kernel == SPTRSV_K_SCALAR_DCSR || I.kernel == SPTRSV_K_VECTOR_DCSR) ? SPTRSV_FMT_DCSR
                                                                                        : SPTRSV_FMT_CSR;
    }
    // storage
    bool dcsr = g.kind == 1 && I.format == SPTRSV_FMT_DCSR;
    S.ci.resize((size_t)tot);
    S.val.resize((size_t)tot * vb);
    if (dcsr) {
      S.nzr = (int32_t)(m - empty);
      S.rows.resize(S.nzr);
      S.rp.assign((size_t)S.nzr + 1, 0);
    } else {
      S.nzr = m;
    }
    // row pointers (serial prefix), then the entries in parallel: every
    // stored row is scaled by 1/d_i (triangles: l_ij/d_i, squares: a_ij/d_i;
    // permute-in scales b the same way), so the solve evaluates
    // x_i = b_i/d_i - sum_j (l_ij/d_i) x_j with no division on the chain
    std::vector<int32_t> slot;  // DCSR: stored-row index of local row k
    {
      int64_t o = 0;
      int32_t jr = 0;
      if (dcsr) slot.assign((size_t)m, -1);
      for (int32_t k = 0; k < m; ++k) {
        int64_t c = hi_idx[k] - lo_idx[k];
        if (dcsr) {
          if (c == 0) continue;
          S.rows[jr] = g.r0 + k;
          slot[k] = jr;
          o += c;
          S.rp[++jr] = (int32_t)o;
        } else {
          o += c;
          S.rp[k + 1] = (int32_t)o;
        }
      }
    }
    parallel_for(m, inner, [&](int64_t ka, int64_t kb) {
      for (int64_t k = ka; k < kb; ++k) {
        int64_t a = lo_idx[k], b = hi_idx[k];
        if (b == a) continue;
        const int64_t o = dcsr ? S.rp[slot[k]] : S.rp[k];
        std::memcpy(&S.ci[o], &p.p_ci[a], (size_t)(b - a) * 4);
        const int32_t r = g.r0 + (int32_t)k;
        if (vb == 8) {
          double d = *(const double*)&p.diag_new[(size_t)r * 8];
          for (int64_t q = a; q < b; ++q) {
            double v = *(const double*)&p.p_val[(size_t)q * 8] / d;
            std::memcpy(&S.val[(size_t)(o + q - a) * 8], &v, 8);
          }
        } else {
          double d = (double)*(const float*)&p.diag_new[(size_t)r * 4];
          for (int64_t q = a; q < b; ++q) {
            float v = (float)((double)*(const float*)&p.p_val[(size_t)q * 4] / d);
            std::memcpy(&S.val[(size_t)(o + q - a) * 4], &v, 4);
          }
        }
      }
    });
  };
  // few segments: one after the other, each with every thread on its rows;
  // many: one thread per segment
  if (threads > 1 && (int)geo.size() >= threads) {
    std::vector<std::thread> th;
    int T = threads;
    for (int t = 0; t < T; ++t)
      th.emplace_back([&, t] {
        for (size_t k = t; k < geo.size(); k += T) build_seg(k, 1);
      });
    for (auto& x : th) x.join();
  } else {
    for (size_t k = 0; k < geo.size(); ++k) build_seg(k, threads);
  }
  return {SPTRSV_SUCCESS, ""};
}

// Which sm_100a kernel runs each segment.  PAPER: the Alg 7 label's own kernel
// (L247-L250).  B200: a cost model over the same features.
void choose_impls(Plan& p) {
  for (auto& S : p.segs) {
    auto& I = S.info;
    if (I.kind == 0) {
      int impl;
      switch (I.kernel) {
        case SPTRSV_K_COMPLETELY_PARALLEL: impl = SPTRSV_IMPL_TRI_DIAG; break;
        case SPTRSV_K_LEVEL_SET: impl = SPTRSV_IMPL_TRI_LEVELSET; break;
        case SPTRSV_K_NEAR_SERIAL: impl = SPTRSV_IMPL_TRI_CHAIN; break;
        default: impl = SPTRSV_IMPL_TRI_SYNCFREE; break;
      }
      const int64_t npieces = S.npieces;
      const bool supernodal = npieces > 0 && (double)(I.row1 - I.row0) / (double)npieces >= 8.0;
      if (p.opts.selector == SPTRSV_SELECT_B200 && I.nlevels > 1 && supernodal) {
        impl = SPTRSV_IMPL_TRI_SUPERNODE;
      } else if (p.opts.selector == SPTRSV_SELECT_B200 && I.nlevels > 1) {
        // B200 thresholds re-derived with the paper's own method (Sec 3.4,
        // L254-L263; scripts/fig5_derive.py -> profiles/r02_fig5.json,
        // DESIGN.md sec. 6.1): every kernel timed on sub-matrices of the five
        // families, the fastest per feature cell.
        //  - the strand wavefront wins on long chains of narrow levels with
        //    few dependencies (C2-like: >= 128 levels);
        //  - the single-CTA chain wins on small triangles (<= 8192 rows)
        //    with >= 32 levels (no cross-SM hop per level);
        //  - everywhere else the mixed sync-free kernel -- including the few-
        //    level triangles the paper gives to level-set (one launch per
        //    level loses to it on B200 at every sampled size); with several
        //    RHS a <= 20-level triangle still runs level by level (exec.cu)
        const int64_t m = I.row1 - I.row0;
        const bool narrow = I.max_level_rows <= 2048 || (m / std::max(1, I.nlevels)) <= 256;
        const int32_t kmax = S.kmax_indeg;
        if (narrow && kmax >= 1 && kmax <= 8 && m >= 4096 && I.nlevels >= 128 &&
            std::getenv("SPTRSV_NO_WAVE") == nullptr)
          impl = SPTRSV_IMPL_TRI_PIPE;
        else if (narrow && m <= 8192 && I.nlevels >= 32)
          impl = SPTRSV_IMPL_TRI_CHAIN;
        else
          impl = SPTRSV_IMPL_TRI_SYNCFREE;
      }
      if (p.opts.force_tri_impl >= SPTRSV_IMPL_TRI_LEVELSET && p.opts.force_tri_impl <= SPTRSV_IMPL_TRI_CHAIN)
        impl = p.opts.force_tri_impl;
      if (p.opts.force_tri_impl == SPTRSV_IMPL_TRI_SUPERNODE && I.nlevels > 1) impl = SPTRSV_IMPL_TRI_SUPERNODE;
      if (p.opts.force_tri_impl == SPTRSV_IMPL_TRI_PIPE && I.nlevels > 1) impl = SPTRSV_IMPL_TRI_PIPE;
      // the level-set and chain kernels walk levels as contiguous row ranges,
      // which only the level-set reordering guarantees; without it a triangle
      // runs sync-free (or supernodal), whatever its Alg 7 label
      if (p.reorder_eff == 1 &&
          (impl == SPTRSV_IMPL_TRI_LEVELSET || impl == SPTRSV_IMPL_TRI_CHAIN || impl == SPTRSV_IMPL_TRI_PIPE))
        impl = supernodal ? SPTRSV_IMPL_TRI_SUPERNODE : SPTRSV_IMPL_TRI_SYNCFREE;
      if (p.opts.force_tri_impl == SPTRSV_IMPL_TRI_DIAG && I.nlevels <= 1) impl = SPTRSV_IMPL_TRI_DIAG;
      I.impl = impl;
    } else {
      int impl = (I.kernel == SPTRSV_K_VECTOR_CSR || I.kernel == SPTRSV_K_VECTOR_DCSR) ? SPTRSV_IMPL_SQ_VECTOR
                                                                                      : SPTRSV_IMPL_SQ_SCALAR;
      // B200: every square streams through the nnz-balanced row-block kernel
      // (the Alg 7 label still fixes the format, CSR or DCSR)
      if (p.opts.selector == SPTRSV_SELECT_B200 && std::getenv("SPTRSV_NO_SQ_ADAPT") == nullptr) impl = SPTRSV_IMPL_SQ_ADAPT;
      if (p.opts.force_sq_impl == SPTRSV_IMPL_SQ_SCALAR || p.opts.force_sq_impl == SPTRSV_IMPL_SQ_VECTOR ||
          p.opts.force_sq_impl == SPTRSV_IMPL_SQ_ADAPT)
        impl = p.opts.force_sq_impl;
      I.impl = impl;
    }
  }
}

int64_t default_min_block_rows(const Plan& p) { return min_block_rows_rule(p); }

}  // namespace sptrsv
