// Device-resident preprocessing: the analysis of
// sptrsv_analyse run on the GPU when the CSR is given in device memory.
// Same readings, same results as the host analysis (analyse.cpp), bit for bit:
//   validate            one thread per row, the LOWEST failing row's first
//                       failing check wins (atomicMin over (row, code))
//   J U J               UPPER input reversed on the device (reading R19)
//   levels              Alg 2 as a sync-free (max,+) sweep
//                       -- the in-degree idea of Alg 3 (L109-L125) with max in
//                       place of +: a row's level is final once every
//                       dependency inside the node has published its own
//   reorder             a stable radix sort of each node's rows by level
//                       (ties keep the current order, reading R4; Sec 3.3
//                       L231-L233); top children inherit (reading R3)
//   P L P^T             mapped columns, one stable segmented sort per row
//   blocks + Alg 7      per-segment row bounds, counts, features (Sec 3.4
//                       L252-L296), CSR / DCSR written straight into the plan
//                       arena, scaled by 1/d (R27)
// When a segment's kernel needs a host-built format (strand wavefront, TMA /
// ELL chain, supernode packing), P L P^T is brought to the host and the host
// extraction + upload finish the plan (still with the device's levels and
// permutation).
#include <cuda_runtime.h>

#include <cub/cub.cuh>

#include <algorithm>
#include <cstring>
#include <numeric>
#include <string>
#include <mutex>
#include <thread>

#include "internal.h"
#include "kernels.cuh"

namespace sptrsv {

Error upload(Plan& p, void* stream);
int count_launches_public(const Plan& p);
void build_sq_items(Segment& S);
SpmmCfg spmm_cfg_public();
int64_t default_min_block_rows(const Plan& p);
void build_sf_items(Segment& S, int32_t& part_base, int selector);
void fuse_square_items(Segment& T, Segment& Q);
bool watchdog_word_acquire(int32_t** h, int32_t** d);
Error prepare_solve_public(Plan& p, int nrhs, cudaStream_t s);

#define DV_TRY(x)                                                                    \
  do {                                                                               \
    cudaError_t e_ = (x);                                                            \
    if (e_ != cudaSuccess)                                                           \
      return Error{SPTRSV_ERROR_CUDA, std::string(#x) + ": " + cudaGetErrorString(e_)}; \
  } while (0)

namespace dv {

enum : int { E_NONE = 0, E_MONO = 1, E_RANGE = 2, E_UNSORTED = 3, E_NOT_TRI = 4, E_MISSING = 5, E_ZERO = 6 };

inline unsigned nblk(int64_t n, int b = 256) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>((n + b - 1) / b, 1 << 20)); }

template <typename T>
__global__ void validate(int n, int64_t nnz, const int* __restrict__ rp, const int* __restrict__ ci,
                         const T* __restrict__ val, int upper, unsigned long long* best) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    int code = E_NONE;
    const int64_t s = rp[i], e = rp[i + 1];
    if (e < s || e > nnz || s < 0) {
      code = E_MONO;
    } else {
      for (int64_t q = s; q < e && !code; ++q) {
        const int c = ci[q];
        if (c < 0 || c >= n) code = E_RANGE;
        else if (q > s && c <= ci[q - 1]) code = E_UNSORTED;
      }
      if (!code) {
        if (!upper) {
          if (e > s && ci[e - 1] > i) code = E_NOT_TRI;
          else if (e == s || ci[e - 1] != i) code = E_MISSING;
          else if (val[e - 1] == T(0)) code = E_ZERO;
        } else {
          if (e > s && ci[s] < i) code = E_NOT_TRI;
          else if (e == s || ci[s] != i) code = E_MISSING;
          else if (val[s] == T(0)) code = E_ZERO;
        }
      }
    }
    if (code) atomicMin(best, ((unsigned long long)i << 8) | (unsigned long long)code);
  }
}

// J U J: row r of the result is row n-1-r of U read backwards (reading R19)
__global__ void rev_len(int n, const int* __restrict__ rp, int* __restrict__ len) {
  for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < n; r += gridDim.x * blockDim.x) {
    const int i = n - 1 - r;
    len[r] = rp[i + 1] - rp[i];
  }
}
template <typename T>
__global__ void juj(int n, const int* __restrict__ rp, const int* __restrict__ ci, const T* __restrict__ val,
                    const int* __restrict__ lrp, int* __restrict__ lci, T* __restrict__ lval) {
  const int lane = threadIdx.x & 31;
  for (int r = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < n; r += (gridDim.x * blockDim.x) >> 5) {
    const int i = n - 1 - r, s = rp[i], e = rp[i + 1], o = lrp[r];
    for (int k = lane; k < e - s; k += 32) {
      lci[o + k] = n - 1 - ci[e - 1 - k];
      lval[o + k] = val[e - 1 - k];
    }
  }
}

__device__ __forceinline__ int ld_lev(const int* p) {
  int v;
  asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_lev(int* p, int v) {
  asm volatile("st.relaxed.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// Alg 2's levels of rows [lo, hi) of the current P L P^T (only dependencies
// inside the node count, reading R5) by a sync-free (max,+) sweep: warps
// claim 32 rows in row order (every dependency precedes its row, so it was
// claimed earlier: no deadlock); a lane whose dependency has not published
// its level keeps its position and retries on the next pass (non-blocking).
// lev (m entries) must hold -1; nlev receives max level + 1.
__global__ void __launch_bounds__(256) level_sweep(int lo, int hi, const int* __restrict__ perm,
                                                   const int* __restrict__ o2n, int identity,
                                                   const int* __restrict__ rp, const int* __restrict__ ci,
                                                   int* __restrict__ lev, unsigned* ticket, int* nlev) {
  constexpr int U = 8;  // dependencies per batch, all loads in flight together
  const int lane = threadIdx.x & 31, m = hi - lo;
  int mx = 0;
  for (;;) {
    int base = 0;
    if (lane == 0) base = (int)atomicAdd(ticket, 32u);
    base = __shfl_sync(0xffffffffu, base, 0);
    if (base >= m) break;
    const int k = base + lane;
    bool done = k >= m;
    int q = 0, e = 0, lv = 0, cnt = 0;
    if (!done) {
      const int o = identity ? lo + k : perm[lo + k];
      q = rp[o];
      e = rp[o + 1] - 1;  // off-diagonals (the diagonal is last)
    }
    int c[U], v[U];
    uint32_t pend = 0;
    bool have = false;
    for (;;) {
      if (!done) {
        for (;;) {
          if (have) {
            if (pend) break;
#pragma unroll
            for (int u = 0; u < U; ++u)
              if (u < cnt && c[u] >= lo) lv = max(lv, v[u] + 1);
            q += cnt;
            have = false;
          }
          if (q >= e) {
            st_lev(lev + k, lv);
            mx = max(mx, lv + 1);
            done = true;
            break;
          }
          cnt = min(U, e - q);
#pragma unroll
          for (int u = 0; u < U; ++u)
            if (u < cnt) c[u] = ci[q + u];
          if (!identity) {
#pragma unroll
            for (int u = 0; u < U; ++u)
              if (u < cnt) c[u] = o2n[c[u]];
          }
#pragma unroll
          for (int u = 0; u < U; ++u)
            if (u < cnt && c[u] >= lo) v[u] = ld_lev(lev + (c[u] - lo));
          pend = 0;
#pragma unroll
          for (int u = 0; u < U; ++u)
            if (u < cnt && c[u] >= lo && v[u] < 0) pend |= 1u << u;
          have = true;
        }
      }
      if (__all_sync(0xffffffffu, done)) break;
      unsigned ns = 0;
      for (;;) {  // lean wait on the pending dependencies of every lane
        if (!done && pend) {
#pragma unroll
          for (int u = 0; u < U; ++u)
            if (pend & (1u << u)) v[u] = ld_lev(lev + (c[u] - lo));
#pragma unroll
          for (int u = 0; u < U; ++u)
            if ((pend & (1u << u)) && v[u] >= 0) pend &= ~(1u << u);
        }
        if (__any_sync(0xffffffffu, !done && !pend)) break;
        ns = ns ? min(ns * 2u, 256u) : 32u;  // back off: keep L2 free for the rows that can advance
        __nanosleep(ns);
      }
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  if (lane == 0 && mx > 0) atomicMax(nlev, mx);
}

__global__ void iota(int m, int* __restrict__ a) {
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < m; k += gridDim.x * blockDim.x) a[k] = k;
}
__global__ void fill_i(int64_t m, int* __restrict__ a, int v) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x)
    a[k] = v;
}

// apply a node's stable sort: rows [lo, lo+m) in sorted order
__global__ void apply_sort(int lo, int m, const int* __restrict__ sidx, const int* __restrict__ slev,
                           const int* __restrict__ perm_old, int* __restrict__ perm, int* __restrict__ o2n,
                           int* __restrict__ lev) {
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < m; k += gridDim.x * blockDim.x) {
    const int old = perm_old[sidx[k]];
    perm[lo + k] = old;
    o2n[old] = lo + k;
    lev[lo + k] = slev[k];
  }
}
__global__ void copy_lev(int lo, int m, const int* __restrict__ l, int* __restrict__ lev) {
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < m; k += gridDim.x * blockDim.x) lev[lo + k] = l[k];
}

// features for the depth retune (R30): widest level, off-diagonal count range
__global__ void level_hist(int n, const int* __restrict__ lev, int* __restrict__ cnt) {
  for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < n; r += gridDim.x * blockDim.x) atomicAdd(cnt + lev[r], 1);
}
__global__ void maxmin(int64_t n, const int* __restrict__ a, int stride_diff, int* out /* {min, max} */) {
  int lo = INT_MAX, hi = INT_MIN;
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
    const int v = stride_diff ? a[k + 1] - a[k] - 1 : a[k];
    lo = min(lo, v);
    hi = max(hi, v);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, o));
    hi = max(hi, __shfl_xor_sync(0xffffffffu, hi, o));
  }
  if ((threadIdx.x & 31) == 0) {
    atomicMin(out, lo);
    atomicMax(out + 1, hi);
  }
}

// fundamental supernodes (reading R29): row r extends row r-1's supernode
// iff its off-diagonal columns are r-1's plus r-1 itself.  rp/ci describe
// the off-diagonal entries of every row: row r's are [a[r], a[r] + l[r]).
__device__ __forceinline__ bool sn_join(int r, const int* __restrict__ a, const int* __restrict__ l,
                                        const int* __restrict__ ci, int gr) {
  const int a0 = a[r - 1], l0 = l[r - 1], a1 = a[r], l1 = l[r];
  if (l1 != l0 + 1 || ci[a1 + l1 - 1] != gr - 1) return false;
  for (int q = 0; q < l0; ++q)
    if (ci[a0 + q] != ci[a1 + q]) return false;
  return true;
}
// pieces of <= 32 rows: every fundamental run of L rows gives ceil(L/32)
__global__ void sn_pieces(int m, int r0g, const int* __restrict__ a, const int* __restrict__ l,
                          const int* __restrict__ ci, unsigned long long* np) {
  unsigned long long c = 0;
  for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < m; r += gridDim.x * blockDim.x) {
    if (r > 0 && sn_join(r, a, l, ci, r0g + r)) continue;
    int len = 1;
    while (r + len < m && sn_join(r + len, a, l, ci, r0g + r + len)) ++len;
    c += (unsigned long long)((len + 31) / 32);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(np, c);
}
// {start, off-diagonal length} of every row of a CSR whose diagonal is last
__global__ void offdiag_al(int n, const int* __restrict__ rp, int* __restrict__ a, int* __restrict__ l) {
  for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < n; r += gridDim.x * blockDim.x) {
    a[r] = rp[r];
    l[r] = rp[r + 1] - rp[r] - 1;
  }
}

// P L P^T
__global__ void plpt_len(int n, const int* __restrict__ perm, const int* __restrict__ rp, int* __restrict__ len) {
  for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < n; r += gridDim.x * blockDim.x) {
    const int o = perm[r];
    len[r] = rp[o + 1] - rp[o];
  }
}
__global__ void plpt_gather(int n, const int* __restrict__ perm, const int* __restrict__ o2n,
                            const int* __restrict__ rp, const int* __restrict__ ci, const int* __restrict__ prp,
                            int* __restrict__ pci, int* __restrict__ src) {
  const int lane = threadIdx.x & 31;
  for (int r = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < n; r += (gridDim.x * blockDim.x) >> 5) {
    const int o = perm[r], s = rp[o], len = rp[o + 1] - s, d = prp[r];
    for (int k = lane; k < len; k += 32) {
      pci[d + k] = o2n[ci[s + k]];
      src[d + k] = s + k;
    }
  }
}
template <typename T>
__global__ void gather_vals(int64_t nnz, const int* __restrict__ src, const T* __restrict__ val, T* __restrict__ out) {
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < nnz; q += (int64_t)gridDim.x * blockDim.x)
    out[q] = val[src[q]];
}
// diagonal (last in its row) and its inverse, as the host computes them
template <typename T>
__global__ void diag_inv(int n, const int* __restrict__ prp, const T* __restrict__ pval, T* __restrict__ diag,
                         T* __restrict__ rdiag) {
  for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < n; r += gridDim.x * blockDim.x) {
    const T d = pval[prp[r + 1] - 1];
    diag[r] = d;
    rdiag[r] = (T)(1.0 / (double)d);
  }
}
// perm in original indexing (UPPER composed with J) and its inverse
__global__ void final_perm(int n, int upper, const int* __restrict__ perm, int* __restrict__ out_perm,
                           int* __restrict__ out_iperm) {
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < n; k += gridDim.x * blockDim.x) {
    const int v = upper ? n - 1 - perm[k] : perm[k];
    out_perm[k] = v;
    out_iperm[v] = k;
  }
}

// per-segment row bounds [lo, lo + cnt) of the entries in cols [c0, c1)
// (TRI: [c0, r), the off-diagonals) -- binary search in the sorted row
__global__ void seg_bounds(int r0, int m, int c0, int c1, int tri, const int* __restrict__ prp,
                           const int* __restrict__ pci, int* __restrict__ lo, int* __restrict__ cnt) {
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < m; k += gridDim.x * blockDim.x) {
    const int r = r0 + k, cend = tri ? r : c1;
    int a = prp[r], b = prp[r + 1];
    int x = a, y = b;  // first >= c0
    while (x < y) {
      const int mid = (x + y) >> 1;
      if (pci[mid] < c0) x = mid + 1;
      else y = mid;
    }
    const int s = x;
    y = b;  // first >= cend
    while (x < y) {
      const int mid = (x + y) >> 1;
      if (pci[mid] < cend) x = mid + 1;
      else y = mid;
    }
    lo[k] = s;
    cnt[k] = x - s;
  }
}
struct SegStat {
  unsigned long long tot;
  int empty, kmax, nl, pad;
  unsigned long long npieces;
};
__global__ void seg_stats(int m, const int* __restrict__ cnt, SegStat* st) {
  unsigned long long tot = 0;
  int empty = 0, kmax = 0;
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < m; k += gridDim.x * blockDim.x) {
    const int c = cnt[k];
    tot += c;
    empty += c == 0;
    kmax = max(kmax, c);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    tot += __shfl_xor_sync(0xffffffffu, tot, o);
    empty += __shfl_xor_sync(0xffffffffu, empty, o);
    kmax = max(kmax, __shfl_xor_sync(0xffffffffu, kmax, o));
  }
  if ((threadIdx.x & 31) == 0) {
    atomicAdd(&st->tot, tot);
    atomicAdd(&st->empty, empty);
    atomicMax(&st->kmax, kmax);
  }
}
__global__ void range_max(int lo, int m, const int* __restrict__ lev, int* out) {
  int mx = -1;
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < m; k += gridDim.x * blockDim.x) mx = max(mx, lev[lo + k]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  if ((threadIdx.x & 31) == 0) atomicMax(out, mx);
}
// level_ptr of a leaf: counts then an exclusive scan (levels are sorted by the reorder)
__global__ void lev_count(int lo, int m, const int* __restrict__ lev, int* __restrict__ lp) {
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < m; k += gridDim.x * blockDim.x) atomicAdd(lp + lev[lo + k] + 1, 1);
}
// DCSR: stored rows and their pointers from the CSR offsets (offs = exclusive scan of cnt)
__global__ void dcsr_rows(int r0, int m, const int* __restrict__ cnt, const int* __restrict__ offs,
                          const int* __restrict__ slot, int* __restrict__ rows, int* __restrict__ srp) {
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < m; k += gridDim.x * blockDim.x)
    if (cnt[k] > 0) {
      rows[slot[k]] = r0 + k;
      srp[slot[k]] = offs[k];
    }
  if (blockIdx.x == 0 && threadIdx.x == 0) srp[slot[m]] = offs[m];
}
__global__ void nonempty(int m, const int* __restrict__ cnt, int* __restrict__ f) {
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < m; k += gridDim.x * blockDim.x) f[k] = cnt[k] > 0;
  if (blockIdx.x == 0 && threadIdx.x == 0) f[m] = 0;
}
// the entries: global permuted columns, values scaled by 1/d_r (R27)
template <typename T>
__global__ void seg_fill(int r0, int m, const int* __restrict__ lo, const int* __restrict__ cnt,
                         const int* __restrict__ offs, const int* __restrict__ pci, const T* __restrict__ pval,
                         const T* __restrict__ diag, int* __restrict__ sci, T* __restrict__ sval) {
  const int lane = threadIdx.x & 31;
  for (int k = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; k < m; k += (gridDim.x * blockDim.x) >> 5) {
    const int a = lo[k], c = cnt[k], o = offs[k];
    if (!c) continue;
    const double d = (double)diag[r0 + k];
    for (int q = lane; q < c; q += 32) {
      sci[o + q] = pci[a + q];
      sval[o + q] = (T)((double)pval[a + q] / d);
    }
  }
}
// supernode pieces of a triangle's own entries: rows' {start, length} in P L P^T
__global__ void tri_al(int m, const int* __restrict__ lo, const int* __restrict__ cnt, int* __restrict__ a,
                       int* __restrict__ l) {
  for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < m; k += gridDim.x * blockDim.x) {
    a[k] = lo[k];
    l[k] = cnt[k];
  }
}

}  // namespace dv

namespace {

// bump allocator over one scratch allocation (released at the end of the analysis)
struct Scratch {
  Plan* p = nullptr;
  char* base = nullptr;
  size_t cap = 0, off = 0;
  cudaStream_t s = nullptr;
  template <typename X>
  X* take(size_t count) {
    size_t o = (off + 255) / 256 * 256;
    off = o + count * sizeof(X);
    return off <= cap ? (X*)(base + o) : nullptr;
  }
};

template <typename T>
Error analyse_device_t(Plan& p, int32_t n, int64_t nnz, const int32_t* d_rp, const int32_t* d_ci, const T* d_val,
                       cudaStream_t s) {
  PhaseClock clk;
  const size_t vb = sizeof(T);
  const bool upper = p.fill == SPTRSV_UPPER;
  // ---- row_ptr ends (host checks, as the host analysis) ----
  int32_t ends[2] = {0, 0};
  DV_TRY(cudaMemcpyAsync(&ends[0], d_rp, 4, cudaMemcpyDeviceToHost, s));
  DV_TRY(cudaMemcpyAsync(&ends[1], d_rp + n, 4, cudaMemcpyDeviceToHost, s));
  DV_TRY(cudaStreamSynchronize(s));
  if (ends[0] != 0) return {SPTRSV_ERROR_INVALID_VALUE, "row_ptr[0] != 0"};
  if ((int64_t)ends[1] != nnz) return {SPTRSV_ERROR_INVALID_VALUE, "nnz != row_ptr[n]"};
  // ---- scratch: one allocation for every temporary of the analysis ----
  const size_t nn = (size_t)std::max(1, n);
  const size_t ne = (size_t)std::max<int64_t>(1, nnz);
  size_t cub_bytes = 0;
  {
    size_t t1 = 0, t2 = 0, t3 = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, t1, (int*)nullptr, (int*)nullptr, (int*)nullptr, (int*)nullptr, n);
    cub::DeviceScan::ExclusiveSum(nullptr, t2, (int*)nullptr, (int*)nullptr, n + 1);
    cub::DeviceSegmentedSort::StableSortPairs(nullptr, t3, (int*)nullptr, (int*)nullptr, (int*)nullptr,
                                              (int*)nullptr, (int)ne, n, (int*)nullptr, (int*)nullptr);
    cub_bytes = std::max({t1, t2, t3}) + 256;
  }
  // geometry at the paper-rule depth bounds the per-segment row arrays (the
  // R30 retune can only lower the depth)
  int64_t rows_tot_max = 0;
  int32_t depth0 = 0;
  {
    const int64_t T0 = p.opts.min_block_rows > 0 ? p.opts.min_block_rows : (int64_t)20 * p.sm_count * 128;
    if (p.opts.depth >= 0) {
      depth0 = 0;
      if (n > 1) {
        int32_t lg = 0;
        while ((int64_t(1) << (lg + 1)) <= n) ++lg;
        depth0 = std::min(p.opts.depth, lg);
      }
    } else if (n) {
      while (((int64_t)n >> (depth0 + 1)) >= T0) ++depth0;
    }
    std::vector<std::pair<int32_t, int32_t>> lv = {{0, n}};
    for (int d = 0; d < depth0; ++d) {
      std::vector<std::pair<int32_t, int32_t>> nx;
      for (auto& nd : lv) {
        const int32_t mid = nd.first + (nd.second - nd.first) / 2;
        nx.push_back({nd.first, mid});
        nx.push_back({mid, nd.second});
      }
      lv.swap(nx);
    }
    for (auto& g : segment_geometry(n, depth0, p.opts.variant, lv)) rows_tot_max += g.r1 - g.r0 + 1;
  }
  if (rows_tot_max > 16 * (int64_t)nn + 64)
    return {SPTRSV_ERROR_NOT_SUPPORTED, "device analysis: segment rows exceed 16 n (use the host analysis)"};
  const size_t nseg_max = ((size_t)2 << std::min(depth0, 24)) + 8;
  size_t need = 0;
  need += (14 * (nn + 2) + 5 * ((size_t)rows_tot_max + nseg_max) + 2 * (nn + 2 * nseg_max + 64)) * 4;
  need += 5 * (ne + 1) * 4;           // P L P^T columns / sources (+ J U J columns)
  need += 2 * ne * vb + 2 * nn * vb;  // P L P^T values (+ J U J values), diag, 1/d
  need += 4 * (nn + 2) + cub_bytes + 64 * 1024 + 64 * 256;
  Scratch S;
  S.p = &p;
  S.s = s;
  S.cap = need;
  S.base = (char*)dalloc(p, need, s);
  if (!S.base) return {SPTRSV_ERROR_ALLOC, "analysis scratch allocation failed (" + std::to_string(need) + " bytes)"};
  struct Free {
    Plan& p;
    Scratch& S;
    ~Free() { dfree(p, S.base, S.s); }
  } free_scratch{p, S};
  unsigned long long* d_err = S.take<unsigned long long>(8);
  int* d_small = S.take<int>(64);
  void* d_cub = S.take<char>(cub_bytes);
  // ---- validate ----
  {
    const unsigned long long none = ~0ull;
    DV_TRY(cudaMemcpyAsync(d_err, &none, 8, cudaMemcpyHostToDevice, s));
    dv::validate<T><<<dv::nblk(n), 256, 0, s>>>(n, nnz, d_rp, d_ci, d_val, upper ? 1 : 0, d_err);
    unsigned long long key = 0;
    DV_TRY(cudaMemcpyAsync(&key, d_err, 8, cudaMemcpyDeviceToHost, s));
    DV_TRY(cudaStreamSynchronize(s));
    if (key != ~0ull) {
      const int row = (int)(key >> 8), code = (int)(key & 0xff);
      const std::string r = std::to_string(row);
      switch (code) {
        case dv::E_MONO: return {SPTRSV_ERROR_INVALID_VALUE, "row_ptr not monotone at row " + r};
        case dv::E_RANGE: return {SPTRSV_ERROR_INVALID_VALUE, "column index out of range in row " + r};
        case dv::E_UNSORTED: return {SPTRSV_ERROR_UNSORTED, "columns not strictly increasing in row " + r};
        case dv::E_NOT_TRI:
          return {SPTRSV_ERROR_NOT_TRIANGULAR,
                  std::string(upper ? "entry below the diagonal in row " : "entry above the diagonal in row ") + r};
        case dv::E_MISSING: return {SPTRSV_ERROR_ZERO_PIVOT, "missing diagonal in row " + r};
        default: return {SPTRSV_ERROR_ZERO_PIVOT, "zero diagonal in row " + r};
      }
    }
  }
  clk.lap("dev: validate");
  p.n = n;
  p.nnz = nnz;
  // ---- the lower form ----
  const int32_t *Lrp = d_rp, *Lci = d_ci;
  const T* Lval = d_val;
  if (upper) {
    int* len = S.take<int>(nn + 1);
    int* lrp = S.take<int>(nn + 1);
    int* lci = S.take<int>(ne);
    T* lval = S.take<T>(ne);
    if (!len || !lrp || !lci || !lval) return {SPTRSV_ERROR_ALLOC, "analysis scratch exhausted"};
    dv::rev_len<<<dv::nblk(n), 256, 0, s>>>(n, d_rp, len);
    DV_TRY(cudaMemsetAsync(len + n, 0, 4, s));
    size_t tb = cub_bytes;
    DV_TRY(cub::DeviceScan::ExclusiveSum(d_cub, tb, len, lrp, n + 1, s));
    dv::juj<T><<<dv::nblk((int64_t)n * 32), 256, 0, s>>>(n, d_rp, d_ci, d_val, lrp, lci, lval);
    Lrp = lrp;
    Lci = lci;
    Lval = lval;
  }
  // ---- depth (L299) ----
  p.min_block_rows = default_min_block_rows(p);
  auto depth_rule = [](int64_t nn2, int64_t T2) {
    int32_t d = 0;
    while ((nn2 >> (d + 1)) >= T2) ++d;
    return d;
  };
  auto clamp_depth = [](int64_t nn2, int32_t d) {
    if (nn2 <= 1) return 0;
    int32_t lg = 0;
    while ((int64_t(1) << (lg + 1)) <= nn2) ++lg;
    return std::min(d, lg);
  };
  p.depth = p.opts.depth >= 0 ? clamp_depth(n, p.opts.depth) : (n ? depth_rule(n, p.min_block_rows) : 0);
  if (p.opts.depth < 0 && n && p.min_block_rows != (int64_t)20 * p.sm_count * 128 && p.opts.min_block_rows == 0 &&
      p.depth < depth_rule(n, (int64_t)20 * p.sm_count * 128))
    p.depth_retuned = 3;  // reading R33, as the host does
  int* d_a = S.take<int>(nn + 1);
  int* d_l = S.take<int>(nn + 1);
  // ---- reorder AUTO (R29): mean fundamental-supernode width of the input ----
  p.reorder_eff = p.opts.reorder == 1 ? 1 : 0;
  if (p.opts.reorder == 2 && n > 0) {
    unsigned long long* np = (unsigned long long*)d_small;
    DV_TRY(cudaMemsetAsync(np, 0, 8, s));
    dv::offdiag_al<<<dv::nblk(n), 256, 0, s>>>(n, Lrp, d_a, d_l);
    dv::sn_pieces<<<dv::nblk(n), 256, 0, s>>>(n, 0, d_a, d_l, Lci, np);
    unsigned long long h = 0;
    DV_TRY(cudaMemcpyAsync(&h, np, 8, cudaMemcpyDeviceToHost, s));
    DV_TRY(cudaStreamSynchronize(s));
    p.reorder_eff = (h > 0 && (double)n / (double)h >= 8.0) ? 1 : 0;
  }
  const bool reorder = p.reorder_eff == 0;
  // ---- levels + reorder of every node (R3), top children inherit ----
  int* perm = S.take<int>(nn);
  int* o2n = S.take<int>(nn);
  int* lev = S.take<int>(nn);      // leaf level of every row, current order
  int* llev = S.take<int>(nn);     // a node's sweep output
  int* skey = S.take<int>(nn);
  int* sidx0 = S.take<int>(nn);
  int* sidx = S.take<int>(nn);
  int* pold = S.take<int>(nn);
  dv::iota<<<dv::nblk(n), 256, 0, s>>>(n, perm);
  dv::iota<<<dv::nblk(n), 256, 0, s>>>(n, o2n);
  if (!perm || !o2n || !lev || !llev || !skey || !sidx0 || !sidx || !pold || !d_a || !d_l)
    return {SPTRSV_ERROR_ALLOC, "analysis scratch exhausted"};
  std::vector<std::pair<int32_t, int32_t>> nodes = {{0, n}};
  std::vector<int32_t> leaf_nl;
  unsigned* tick = (unsigned*)(d_small + 8);
  int* nlv = d_small + 9;
  for (int32_t d = 0; d <= p.depth && n > 0; ++d) {
    for (size_t kx = 0; kx < nodes.size(); ++kx) {
      if (d > 0 && kx % 2 == 0) continue;  // a top child: levels and order inherited
      const int lo = nodes[kx].first, hi = nodes[kx].second, m = hi - lo;
      if (m == 0) continue;
      dv::fill_i<<<dv::nblk(m), 256, 0, s>>>(m, llev, -1);
      DV_TRY(cudaMemsetAsync(tick, 0, 8, s));  // ticket and nlev
      const unsigned g = std::min<unsigned>(dv::nblk(m, 256), (unsigned)p.sm_count * 8);
      dv::level_sweep<<<g, 256, 0, s>>>(lo, hi, perm, o2n, d == 0 ? 1 : 0, Lrp, Lci, llev, tick, nlv);
      if (reorder) {
        int nl = 0;
        DV_TRY(cudaMemcpyAsync(&nl, nlv, 4, cudaMemcpyDeviceToHost, s));
        DV_TRY(cudaStreamSynchronize(s));
        int bits = 1;
        while ((1 << bits) < nl) ++bits;
        dv::iota<<<dv::nblk(m), 256, 0, s>>>(m, sidx0);
        size_t tb = cub_bytes;
        DV_TRY(cub::DeviceRadixSort::SortPairs(d_cub, tb, llev, skey, sidx0, sidx, m, 0, bits, s));
        DV_TRY(cudaMemcpyAsync(pold, perm + lo, (size_t)m * 4, cudaMemcpyDeviceToDevice, s));
        dv::apply_sort<<<dv::nblk(m), 256, 0, s>>>(lo, m, sidx, skey, pold, perm, o2n, lev);
      } else {
        dv::copy_lev<<<dv::nblk(m), 256, 0, s>>>(lo, m, llev, lev);
      }
    }
    if (clk.on) clk.lap(("dev:   levels depth " + std::to_string(d)).c_str());
    // depth retune under the B200 selector (reading R30), as the host does
    if (d == 0 && p.depth > 0 && p.opts.depth < 0 && p.opts.min_block_rows == 0 &&
        p.opts.selector == SPTRSV_SELECT_B200 && p.reorder_eff == 0 && n >= 4096 &&
        std::getenv("SPTRSV_NO_DEPTH_RETUNE") == nullptr) {
      int nl = 0;
      DV_TRY(cudaMemcpyAsync(&nl, nlv, 4, cudaMemcpyDeviceToHost, s));
      DV_TRY(cudaStreamSynchronize(s));
      int* cnt = d_a;
      DV_TRY(cudaMemsetAsync(cnt, 0, (size_t)(nl + 1) * 4, s));
      dv::level_hist<<<dv::nblk(n), 256, 0, s>>>(n, lev, cnt);
      int init[4] = {INT_MAX, INT_MIN, INT_MAX, INT_MIN};
      DV_TRY(cudaMemcpyAsync(d_small + 16, init, 16, cudaMemcpyHostToDevice, s));
      dv::maxmin<<<dv::nblk(nl), 256, 0, s>>>(nl, cnt, 0, d_small + 16);
      dv::maxmin<<<dv::nblk(n), 256, 0, s>>>(n, Lrp, 1, d_small + 18);
      int h[4];
      DV_TRY(cudaMemcpyAsync(h, d_small + 16, 16, cudaMemcpyDeviceToHost, s));
      DV_TRY(cudaStreamSynchronize(s));
      const int wmax = h[1], kmax = h[3];
      if (wmax <= 2048 && kmax >= 1 && kmax <= 8) {
        p.depth = 0;
        p.depth_retuned = 1;
      }
    }
    if (d == p.depth) break;
    std::vector<std::pair<int32_t, int32_t>> next;
    for (auto& nd : nodes) {
      int32_t mid = nd.first + (nd.second - nd.first) / 2;  // reading R1
      next.push_back({nd.first, mid});
      next.push_back({mid, nd.second});
    }
    nodes.swap(next);
  }
  // levels per leaf
  leaf_nl.assign(nodes.size(), 0);
  {
    int* mx = d_small + 24;
    const int nlf = (int)nodes.size();
    std::vector<int> init((size_t)nlf, -1);
    int* dmx = S.take<int>((size_t)nlf);
    DV_TRY(cudaMemcpyAsync(dmx, init.data(), (size_t)nlf * 4, cudaMemcpyHostToDevice, s));
    for (int kx = 0; kx < nlf; ++kx) {
      const int lo = nodes[kx].first, m = nodes[kx].second - lo;
      if (m > 0) dv::range_max<<<std::min<unsigned>(dv::nblk(m), 1024), 256, 0, s>>>(lo, m, lev, dmx + kx);
    }
    DV_TRY(cudaMemcpyAsync(init.data(), dmx, (size_t)nlf * 4, cudaMemcpyDeviceToHost, s));
    DV_TRY(cudaStreamSynchronize(s));
    for (int kx = 0; kx < nlf; ++kx) leaf_nl[kx] = init[kx] + 1;
    (void)mx;
  }
  clk.lap("dev: levels + reorder");
  // ---- P L P^T with sorted columns (R6) ----
  int* prp = S.take<int>(nn + 1);
  const int* pci = Lci;
  const T* pval = Lval;
  if (reorder) {
    int* len = d_a;
    dv::plpt_len<<<dv::nblk(n), 256, 0, s>>>(n, perm, Lrp, len);
    DV_TRY(cudaMemsetAsync(len + n, 0, 4, s));
    size_t tb = cub_bytes;
    DV_TRY(cub::DeviceScan::ExclusiveSum(d_cub, tb, len, prp, n + 1, s));
    int* ci1 = S.take<int>(ne);
    int* src1 = S.take<int>(ne);
    int* ci2 = S.take<int>(ne);
    int* src2 = S.take<int>(ne);
    T* pv = S.take<T>(ne);
    if (!ci1 || !src1 || !ci2 || !src2 || !pv) return {SPTRSV_ERROR_ALLOC, "analysis scratch exhausted"};
    dv::plpt_gather<<<dv::nblk((int64_t)n * 32), 256, 0, s>>>(n, perm, o2n, Lrp, Lci, prp, ci1, src1);
    tb = cub_bytes;
    DV_TRY(cub::DeviceSegmentedSort::StableSortPairs(d_cub, tb, ci1, ci2, src1, src2, (int)nnz, n, prp, prp + 1, s));
    dv::gather_vals<T><<<dv::nblk(nnz), 256, 0, s>>>(nnz, src2, Lval, pv);
    pci = ci2;
    pval = pv;
  } else {
    DV_TRY(cudaMemcpyAsync(prp, Lrp, (size_t)(n + 1) * 4, cudaMemcpyDeviceToDevice, s));
  }
  T* diag = S.take<T>(nn);
  T* rdiag = S.take<T>(nn);
  if (!prp || !diag || !rdiag) return {SPTRSV_ERROR_ALLOC, "analysis scratch exhausted"};
  dv::diag_inv<T><<<dv::nblk(n), 256, 0, s>>>(n, prp, pval, diag, rdiag);
  clk.lap("dev: P L P^T");

  // ---- segments: geometry, bounds, features ----
  const std::vector<SegGeo> geo = segment_geometry(n, p.depth, p.opts.variant, nodes);
  const int nseg = (int)geo.size();
  p.segs.clear();
  p.segs.resize(nseg);
  int64_t rows_tot = 0;
  for (auto& g : geo) rows_tot += g.r1 - g.r0;
  int* blo = S.take<int>((size_t)rows_tot + nseg);
  int* bcnt = S.take<int>((size_t)rows_tot + nseg);
  dv::SegStat* dst = S.take<dv::SegStat>((size_t)std::max(1, nseg));
  if (!blo || !bcnt || !dst) return {SPTRSV_ERROR_ALLOC, "analysis scratch exhausted"};
  DV_TRY(cudaMemsetAsync(dst, 0, sizeof(dv::SegStat) * std::max(1, nseg), s));
  std::vector<int64_t> boff((size_t)nseg + 1, 0);
  for (int i = 0; i < nseg; ++i) boff[i + 1] = boff[i] + (geo[i].r1 - geo[i].r0) + 1;
  for (int i = 0; i < nseg; ++i) {
    const SegGeo& g = geo[i];
    const int m = g.r1 - g.r0;
    if (!m) continue;
    int *lo = blo + boff[i], *cnt = bcnt + boff[i];
    dv::seg_bounds<<<dv::nblk(m), 256, 0, s>>>(g.r0, m, g.c0, g.c1, g.kind == 0, prp, pci, lo, cnt);
    dv::seg_stats<<<std::min<unsigned>(dv::nblk(m), 1024), 256, 0, s>>>(m, cnt, dst + i);
    if (g.kind == 0) {  // supernode pieces of the triangle's own entries (selector feature)
      dv::tri_al<<<dv::nblk(m), 256, 0, s>>>(m, lo, cnt, d_a, d_l);
      dv::sn_pieces<<<dv::nblk(m), 256, 0, s>>>(m, g.r0, d_a, d_l, pci, &dst[i].npieces);
    }
  }
  std::vector<dv::SegStat> hst((size_t)std::max(1, nseg));
  DV_TRY(cudaMemcpyAsync(hst.data(), dst, sizeof(dv::SegStat) * std::max(1, nseg), cudaMemcpyDeviceToHost, s));
  // level_ptr of every leaf triangle
  std::vector<int64_t> lpoff((size_t)nseg + 1, 0);
  for (int i = 0; i < nseg; ++i)
    lpoff[i + 1] = lpoff[i] + (geo[i].kind == 0 ? (int64_t)leaf_nl[geo[i].leaf] + 2 : 0);
  int* dlp = S.take<int>((size_t)std::max<int64_t>(1, lpoff[nseg]));
  int* dlp2 = S.take<int>((size_t)std::max<int64_t>(1, lpoff[nseg]));
  if (!dlp || !dlp2) return {SPTRSV_ERROR_ALLOC, "analysis scratch exhausted"};
  DV_TRY(cudaMemsetAsync(dlp, 0, (size_t)std::max<int64_t>(1, lpoff[nseg]) * 4, s));
  for (int i = 0; i < nseg; ++i)
    if (geo[i].kind == 0 && geo[i].r1 > geo[i].r0) {
      const int m = geo[i].r1 - geo[i].r0, nl = leaf_nl[geo[i].leaf];
      dv::lev_count<<<dv::nblk(m), 256, 0, s>>>(geo[i].r0, m, lev, dlp + lpoff[i]);
      size_t tb = cub_bytes;
      DV_TRY(cub::DeviceScan::InclusiveSum(d_cub, tb, dlp + lpoff[i], dlp2 + lpoff[i], nl + 1, s));
    }
  std::vector<int32_t> hlp((size_t)std::max<int64_t>(1, lpoff[nseg]));
  DV_TRY(cudaMemcpyAsync(hlp.data(), dlp2, hlp.size() * 4, cudaMemcpyDeviceToHost, s));
  DV_TRY(cudaStreamSynchronize(s));
  for (int i = 0; i < nseg; ++i) {
    const SegGeo& g = geo[i];
    Segment& Sg = p.segs[i];
    sptrsv_seg_info_t& I = Sg.info;
    const int m = g.r1 - g.r0;
    I.kind = g.kind;
    I.row0 = g.r0;
    I.row1 = g.r1;
    I.col0 = g.c0;
    I.col1 = g.c1;
    const int64_t tot = (int64_t)hst[i].tot;
    if (g.kind == 0) {
      I.nnz = tot + m;
      I.nnz_per_row = m ? (int32_t)(I.nnz / m) : 0;
      I.nlevels = leaf_nl[g.leaf];
      I.empty_rows = 0;
      I.kernel = select_tri(I.nlevels, I.nnz_per_row);
      I.format = I.kernel == SPTRSV_K_COMPLETELY_PARALLEL ? SPTRSV_FMT_DIAG : SPTRSV_FMT_CSR;
      Sg.level_ptr.assign(hlp.begin() + lpoff[i], hlp.begin() + lpoff[i] + I.nlevels + 1);
      int32_t mx = 0;
      for (int l = 0; l < I.nlevels; ++l) mx = std::max(mx, Sg.level_ptr[l + 1] - Sg.level_ptr[l]);
      I.max_level_rows = mx;
      Sg.nzr = m;
      Sg.kmax_indeg = hst[i].kmax;
      Sg.npieces = (int64_t)hst[i].npieces;
    } else {
      I.nnz = tot;
      I.nnz_per_row = m ? (int32_t)(tot / m) : 0;
      I.empty_rows = hst[i].empty;
      I.nlevels = 0;
      I.kernel = select_sq(I.nnz_per_row, I.empty_rows, m);
      I.format = (I.kernel == SPTRSV_K_SCALAR_DCSR || I.kernel == SPTRSV_K_VECTOR_DCSR) ? SPTRSV_FMT_DCSR
                                                                                        : SPTRSV_FMT_CSR;
      Sg.nzr = I.format == SPTRSV_FMT_DCSR ? m - I.empty_rows : m;
    }
  }
  choose_impls(p);
  clk.lap("dev: segments + Alg 7");
  bool device_formats = true;  // every segment's kernel runs on plain CSR / DCSR (+ items)
  for (auto& Sg : p.segs)
    if (Sg.info.kind == 0 && (Sg.info.impl == SPTRSV_IMPL_TRI_CHAIN || Sg.info.impl == SPTRSV_IMPL_TRI_PIPE ||
                              Sg.info.impl == SPTRSV_IMPL_TRI_SUPERNODE))
      device_formats = false;
  if (!device_formats) {
    // ---- host-built formats: bring P L P^T, the permutation and the leaf
    // levels to the host and finish with the host extraction + upload ----
    p.p_rp.assign((size_t)n + 1, 0);
    std::vector<int32_t> hrp((size_t)n + 1);
    std::vector<int32_t> hperm(nn);
    p.p_ci.resize((size_t)nnz);
    p.p_val.resize((size_t)nnz * vb);
    p.leaf_level.resize(n);
    p.diag_new.resize((size_t)n * vb);
    p.rdiag_new.resize((size_t)n * vb);
    DV_TRY(cudaMemcpyAsync(hrp.data(), prp, (size_t)(n + 1) * 4, cudaMemcpyDeviceToHost, s));
    DV_TRY(cudaMemcpyAsync(p.p_ci.data(), pci, (size_t)nnz * 4, cudaMemcpyDeviceToHost, s));
    DV_TRY(cudaMemcpyAsync(p.p_val.data(), pval, (size_t)nnz * vb, cudaMemcpyDeviceToHost, s));
    DV_TRY(cudaMemcpyAsync(p.leaf_level.data(), lev, nn * 4, cudaMemcpyDeviceToHost, s));
    DV_TRY(cudaMemcpyAsync(hperm.data(), perm, nn * 4, cudaMemcpyDeviceToHost, s));
    DV_TRY(cudaMemcpyAsync(p.diag_new.data(), diag, (size_t)n * vb, cudaMemcpyDeviceToHost, s));
    DV_TRY(cudaMemcpyAsync(p.rdiag_new.data(), rdiag, (size_t)n * vb, cudaMemcpyDeviceToHost, s));
    DV_TRY(cudaStreamSynchronize(s));
    for (int r = 0; r <= n; ++r) p.p_rp[r] = hrp[r];
    p.perm.resize(n);
    for (int k = 0; k < n; ++k) p.perm[k] = upper ? n - 1 - hperm[k] : hperm[k];
    p.lower_old = hperm;
    clk.lap("dev: download for host formats");
    int threads = p.opts.threads > 0 ? p.opts.threads : (int)std::max(1u, std::thread::hardware_concurrency());
    threads = std::min(threads, 64);
    Error e = build_segments_host(p, nodes, leaf_nl, threads);
    if (e.status) return e;
    choose_impls(p);
    clk.lap("dev: host segments");
    p.dev_analysed = false;  // host copies are complete
    p.analysis_where = 2;
    return upload(p, (void*)s);
  }

  // ---- device formats: the arena is written on the device ----
  p.dev_analysed = true;
  p.host_ready = false;
  p.analysis_where = 1;
  // host row pointers of every segment (the item builders are host greedy
  // passes over row pointers only)
  std::vector<int64_t> sq_off((size_t)nseg + 1, 0);
  int* offs_all = S.take<int>((size_t)rows_tot + nseg);
  int* nz_all = S.take<int>((size_t)rows_tot + nseg);
  int* slot_all = S.take<int>((size_t)rows_tot + nseg);
  if (!offs_all || !nz_all || !slot_all) return {SPTRSV_ERROR_ALLOC, "analysis scratch exhausted"};
  for (int i = 0; i < nseg; ++i) {
    const int m = geo[i].r1 - geo[i].r0;
    int* cnt = bcnt + boff[i];
    DV_TRY(cudaMemsetAsync(cnt + m, 0, 4, s));
    size_t tb = cub_bytes;
    DV_TRY(cub::DeviceScan::ExclusiveSum(d_cub, tb, cnt, offs_all + boff[i], m + 1, s));
    if (p.segs[i].info.kind == 1 && p.segs[i].info.format == SPTRSV_FMT_DCSR) {
      dv::nonempty<<<dv::nblk(m + 1), 256, 0, s>>>(m, cnt, nz_all + boff[i]);
      tb = cub_bytes;
      DV_TRY(cub::DeviceScan::ExclusiveSum(d_cub, tb, nz_all + boff[i], slot_all + boff[i], m + 1, s));
    }
  }
  // CSR offsets of every segment to the host in ONE copy through a pinned
  // buffer (the item builders are host passes over row pointers)
  std::vector<std::vector<int32_t>> hoffs((size_t)nseg);
  {
    static std::mutex pin_mu;
    static int32_t* pin = nullptr;
    static size_t pin_n = 0;
    std::lock_guard<std::mutex> lk(pin_mu);
    const size_t tot = (size_t)boff[nseg];
    if (tot > pin_n) {
      if (pin) cudaFreeHost(pin);
      pin = nullptr;
      pin_n = 0;
      if (cudaHostAlloc((void**)&pin, tot * 4, cudaHostAllocDefault) != cudaSuccess) {
        cudaGetLastError();
        pin = nullptr;
      } else {
        pin_n = tot;
      }
    }
    std::vector<int32_t> pageable;
    int32_t* hb = pin;
    if (!hb) {
      pageable.resize(tot);
      hb = pageable.data();
    }
    DV_TRY(cudaMemcpyAsync(hb, offs_all, tot * 4, cudaMemcpyDeviceToHost, s));
    DV_TRY(cudaStreamSynchronize(s));
    for (int i = 0; i < nseg; ++i) {
      const int m = geo[i].r1 - geo[i].r0;
      hoffs[i].assign(hb + boff[i], hb + boff[i] + m + 1);
    }
  }
  clk.lap("dev: row pointers to host");
  // stored row pointers on the host (items); DCSR compacts the nonempty rows
  for (int i = 0; i < nseg; ++i) {
    Segment& Sg = p.segs[i];
    const int m = geo[i].r1 - geo[i].r0;
    if (Sg.info.kind == 1 && Sg.info.format == SPTRSV_FMT_DCSR) {
      Sg.rp.clear();
      Sg.rp.reserve((size_t)Sg.nzr + 1);
      for (int k = 0; k < m; ++k)
        if (hoffs[i][k + 1] > hoffs[i][k]) Sg.rp.push_back(hoffs[i][k]);
      Sg.rp.push_back(hoffs[i][m]);
    } else {
      Sg.rp.swap(hoffs[i]);
    }
  }
  // items (host greedy, exactly the host-analysis items), one thread per segment
  p.npart = 0;
  p.nticket = 0;
  p.needs_sentinel = false;
  p.needs_flags = false;
  {
    std::vector<std::thread> th;
    for (int i = 0; i < nseg; ++i) th.emplace_back([&, i] { build_sq_items(p.segs[i]); });
    for (auto& x : th) x.join();
  }
  for (int i = 0; i < nseg; ++i) {  // part slots numbered in order; squares fused as in upload()
    p.segs[i].fused_sq = -1;
    p.segs[i].fused = false;
  }
  for (int i = 0; i < nseg; ++i) build_sf_items(p.segs[i], p.npart, p.opts.selector);
  for (int i = 0; i + 1 < nseg; ++i) {
    Segment& Sg = p.segs[i];
    if (Sg.sf_mixed && std::getenv("SPTRSV_SQ_FUSE")) {
      p.segs[i + 1].dev_dcsr = p.segs[i + 1].info.kind == 1 && p.segs[i + 1].info.format == SPTRSV_FMT_DCSR;
      p.segs[i + 1].dev_nzr = p.segs[i + 1].nzr;
      fuse_square_items(Sg, p.segs[i + 1]);
      if (p.segs[i + 1].fused) Sg.fused_sq = i + 1;
    }
  }
  clk.lap("dev: items");
  // ---- arena layout (as upload(): perm | iperm | 1/d | segments | tickets | ctl | part) ----
  size_t off = 0;
  auto take = [&](size_t bytes) {
    size_t o = off;
    off = (off + bytes + 255) / 256 * 256;
    return o;
  };
  const size_t o_perm = take((size_t)2 * n * 4);
  const size_t o_rdiag = take((size_t)n * vb);
  const size_t o_lev = take((size_t)n * 4);  // leaf levels (introspection of device plans)
  struct Offs { size_t rp, ci, val, rows, lp, sq, sf; };
  std::vector<Offs> so((size_t)nseg);
  for (int i = 0; i < nseg; ++i) {
    Segment& Sg = p.segs[i];
    const auto& I = Sg.info;
    const int64_t nstore = I.kind == 0 ? I.nnz - (I.row1 - I.row0) : I.nnz;
    so[i].rp = take(((size_t)Sg.nzr + 1) * 4);
    so[i].ci = take((size_t)nstore * 4);
    so[i].val = take((size_t)nstore * vb);
    so[i].rows = take(I.kind == 1 && I.format == SPTRSV_FMT_DCSR ? (size_t)Sg.nzr * 4 : 0);
    so[i].lp = take(Sg.level_ptr.size() * 4);
    so[i].sq = take(Sg.sq_items.size() * 4);
    so[i].sf = take(Sg.sf_items.size() * 4);
    if (I.kind == 0) Sg.ticket_slot = p.nticket++;
    if (I.kind == 0 && I.impl == SPTRSV_IMPL_TRI_SYNCFREE) {
      p.needs_sentinel = true;
      p.needs_flags = true;
    }
    Sg.dev_dcsr = I.kind == 1 && I.format == SPTRSV_FMT_DCSR;
    Sg.dev_nzr = Sg.nzr;
  }
  const size_t o_tickets = take((size_t)std::max(1, p.nticket) * 4);
  const size_t o_ctl = take(16);
  const size_t o_part = take((size_t)std::max(1, p.npart) * vb);
  p.arena_bytes = off;
  int dev = 0;
  DV_TRY(cudaGetDevice(&dev));
  p.device = dev;
  p.arena = dalloc(p, std::max<size_t>(off, 256), s);
  if (!p.arena) return {SPTRSV_ERROR_ALLOC, "plan arena allocation failed (" + std::to_string(off) + " bytes)"};
  char* A = (char*)p.arena;
  DV_TRY(cudaMemsetAsync(A, 0, off, s));
  dv::final_perm<<<dv::nblk(n), 256, 0, s>>>(n, upper ? 1 : 0, perm, (int*)(A + o_perm), (int*)(A + o_perm) + n);
  DV_TRY(cudaMemcpyAsync(A + o_rdiag, rdiag, (size_t)n * vb, cudaMemcpyDeviceToDevice, s));
  DV_TRY(cudaMemcpyAsync(A + o_lev, lev, (size_t)n * 4, cudaMemcpyDeviceToDevice, s));
  for (int i = 0; i < nseg; ++i) {
    Segment& Sg = p.segs[i];
    const auto& I = Sg.info;
    const int m = I.row1 - I.row0;
    int *lo = blo + boff[i], *cnt = bcnt + boff[i], *offs = offs_all + boff[i];
    if (m > 0) {
      if (Sg.dev_dcsr)
        dv::dcsr_rows<<<dv::nblk(m), 256, 0, s>>>(I.row0, m, cnt, offs, slot_all + boff[i], (int*)(A + so[i].rows),
                                                  (int*)(A + so[i].rp));
      else
        DV_TRY(cudaMemcpyAsync(A + so[i].rp, offs, (size_t)(m + 1) * 4, cudaMemcpyDeviceToDevice, s));
      dv::seg_fill<T><<<dv::nblk((int64_t)m * 32), 256, 0, s>>>(I.row0, m, lo, cnt, offs, pci, pval, diag,
                                                                 (int*)(A + so[i].ci), (T*)(A + so[i].val));
    }
    DV_TRY(cudaMemcpyAsync(A + so[i].lp, Sg.level_ptr.data(), Sg.level_ptr.size() * 4, cudaMemcpyHostToDevice, s));
    DV_TRY(cudaMemcpyAsync(A + so[i].sq, Sg.sq_items.data(), Sg.sq_items.size() * 4, cudaMemcpyHostToDevice, s));
    DV_TRY(cudaMemcpyAsync(A + so[i].sf, Sg.sf_items.data(), Sg.sf_items.size() * 4, cudaMemcpyHostToDevice, s));
    Sg.d_rp = (const int32_t*)(A + so[i].rp);
    Sg.d_ci = (const int32_t*)(A + so[i].ci);
    Sg.d_val = (const void*)(A + so[i].val);
    Sg.d_rows = (const int32_t*)(A + so[i].rows);
    Sg.d_level_ptr = (const int32_t*)(A + so[i].lp);
    Sg.d_sq_items = (const int32_t*)(A + so[i].sq);
    Sg.d_sf_items = (const int32_t*)(A + so[i].sf);
  }
  p.d_perm = (const int32_t*)(A + o_perm);
  p.d_rdiag = (const void*)(A + o_rdiag);
  p.d_leaf_level = (const int32_t*)(A + o_lev);
  p.d_tickets = (uint32_t*)(A + o_tickets);
  p.d_derr = (int32_t*)(A + o_ctl);
  p.d_epoch = (uint32_t*)(A + o_ctl + 8);
  p.d_part = (void*)(A + o_part);
  if (!watchdog_word_acquire(&p.h_error, &p.d_error)) {
    p.h_error = nullptr;
    p.d_error = nullptr;
  } else {
    *p.h_error = 0;
  }
  if (p.opts.max_nrhs > 0) {
    Error e = prepare_solve_public(p, p.opts.max_nrhs, s);
    if (e.status) return e;
    p.epoch = 0;
  }
  DV_TRY(cudaStreamSynchronize(s));  // the host vectors passed to async copies die with this call
  p.launches_per_solve = count_launches_public(p);
  clk.lap("dev: arena written");
  return {SPTRSV_SUCCESS, ""};
}

}  // namespace

Error analyse_device(Plan& p, int32_t n, int64_t nnz, const int32_t* d_rp, const int32_t* d_ci, const void* d_val,
                     void* stream) {
  p.backoff_ns = 128;
  p.wd_spins = k::kWatchdogSpins;
  if (const char* e = std::getenv("SPTRSV_WATCHDOG_SPINS")) p.wd_spins = (uint32_t)std::max(1024, std::atoi(e));
  p.spmm = spmm_cfg_public();
  if (p.dtype == SPTRSV_R64F)
    return analyse_device_t<double>(p, n, nnz, d_rp, d_ci, (const double*)d_val, (cudaStream_t)stream);
  return analyse_device_t<float>(p, n, nnz, d_rp, d_ci, (const float*)d_val, (cudaStream_t)stream);
}

// Host copies of a device-analysed plan (introspection, plan hash): the
// permutation, the leaf levels, 1/d and every segment's stored arrays.
Error materialize_host(Plan& p) {
  if (p.host_ready) return {SPTRSV_SUCCESS, ""};
  const int n = p.n;
  const size_t vb = p.vbytes;
  DV_TRY(cudaSetDevice(p.device));
  std::vector<int32_t> hp((size_t)2 * n);
  p.perm.resize(n);
  p.leaf_level.resize(n);
  p.rdiag_new.resize((size_t)n * vb);
  DV_TRY(cudaMemcpy(p.perm.data(), p.d_perm, (size_t)n * 4, cudaMemcpyDeviceToHost));
  DV_TRY(cudaMemcpy(p.leaf_level.data(), p.d_leaf_level, (size_t)n * 4, cudaMemcpyDeviceToHost));
  DV_TRY(cudaMemcpy(p.rdiag_new.data(), p.d_rdiag, (size_t)n * vb, cudaMemcpyDeviceToHost));
  p.lower_old.resize(n);
  for (int k = 0; k < n; ++k) p.lower_old[k] = p.fill == SPTRSV_LOWER ? p.perm[k] : n - 1 - p.perm[k];
  for (auto& S : p.segs) {
    const auto& I = S.info;
    const int64_t nstore = I.kind == 0 ? I.nnz - (I.row1 - I.row0) : I.nnz;
    S.ci.resize((size_t)nstore);
    S.val.resize((size_t)nstore * vb);
    if (nstore) {
      DV_TRY(cudaMemcpy(S.ci.data(), S.d_ci, (size_t)nstore * 4, cudaMemcpyDeviceToHost));
      DV_TRY(cudaMemcpy(S.val.data(), S.d_val, (size_t)nstore * vb, cudaMemcpyDeviceToHost));
    }
    if (S.dev_dcsr) {
      S.rows.resize(S.nzr);
      if (S.nzr) DV_TRY(cudaMemcpy(S.rows.data(), S.d_rows, (size_t)S.nzr * 4, cudaMemcpyDeviceToHost));
    }
    if (I.kind == 0) {
      const int m = I.row1 - I.row0;
      S.in_degree.resize(m);
      for (int k = 0; k < m; ++k) S.in_degree[k] = S.rp[k + 1] - S.rp[k];
    }
  }
  p.host_ready = true;
  return {SPTRSV_SUCCESS, ""};
}

}  // namespace sptrsv
