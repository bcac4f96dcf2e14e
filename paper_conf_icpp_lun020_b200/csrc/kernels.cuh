// sm_100a kernels of the recursive-block SpTRSV (Alg 7).
//
// Buffers of one solve, both row-major n x nrhs in the
// permuted order (the nrhs values of a component are contiguous):
//   bw  the right-hand side being updated: permute-in writes D^{-1} P b, every
//       square subtracts A' x from its rows (the paper's SpMV "updating b",
//       L146/L164, with A' = D^{-1} A), every triangle reads its rows once.
//   xs  the solution.  Triangles write x_i = bw_i - sum_j l'_ij x_j with
//       l' = D^{-1} L (scaled by the analysis, so no division sits on the
//       dependency chain); squares read it; permute-out scatters it.
// When a plan has a sync-free triangle, permute-in fills xs with a signalling
// NaN (SENT).  No floating-point operation can produce a signalling NaN, so a
// value that differs from SENT is a solved x_j: the value is its own ready
// flag (one 8-byte store publishes it, one strong load polls AND fetches it;
// no flag array, no release fence, no counter reset).
//
// Memory-ordering facts used (checked in SASS):
//   ld.relaxed.gpu -> LDG.E.STRONG.GPU (served by L2, never a stale L1 line);
//   st.relaxed.gpu -> STG.E.STRONG.GPU;  ld.acquire.gpu would add CCTL.IVALL
//   (a whole-L1 invalidate per poll) and is not needed: the polled word IS
//   the data.
#pragma once
#include <cstdint>

namespace sptrsv {
namespace k {

constexpr uint32_t kWatchdogSpins = 1u << 25;  // ~ seconds of polling

// ---------------------------------------------------------------- sentinel
__device__ __forceinline__ bool is_sent(double v) {
  return __double_as_longlong(v) == (long long)0x7FF4000000000BADull;
}
__device__ __forceinline__ bool is_sent(float v) { return __float_as_uint(v) == 0x7FA00BADu; }
template <typename T>
__device__ __forceinline__ T sent();
template <>
__device__ __forceinline__ double sent<double>() {
  return __longlong_as_double((long long)0x7FF4000000000BADull);
}
template <>
__device__ __forceinline__ float sent<float>() {
  return __uint_as_float(0x7FA00BADu);
}

__device__ __forceinline__ double ld_strong(const double* p) {
  double v;
  asm volatile("ld.relaxed.gpu.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ float ld_strong(const float* p) {
  float v;
  asm volatile("ld.relaxed.gpu.global.f32 %0, [%1];" : "=f"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_strong(double* p, double v) {
  asm volatile("st.relaxed.gpu.global.f64 [%0], %1;" ::"l"(p), "d"(v) : "memory");
}
__device__ __forceinline__ void st_strong(float* p, float v) {
  asm volatile("st.relaxed.gpu.global.f32 [%0], %1;" ::"l"(p), "f"(v) : "memory");
}
template <typename T>
__device__ __forceinline__ T ldg_nc(const T* p) {
  return __ldg(p);
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

struct SolveState {
  uint32_t* tickets;  // per-segment row-claim counters, zeroed by permute-in
  int nticket;
  int* error;         // mapped host word (watchdog)
  uint32_t* flags;    // nrhs > 1: per-row ready flags (global row index), value = epoch when solved
  // Epochs live on the device so a captured solve (CUDA graph) replays
  // correctly: epoch_dev[0] = this solve's first epoch, epoch_dev[1] = the
  // last epoch handed out; permute-in (block 0) advances them by `span`.
  uint32_t* epoch_dev;
  uint32_t epoch_off;   // offset of this launch inside the solve's span (supernodal chunk index)
  uint32_t span;        // epochs this solve uses (0: no flags polled)
  uint32_t backoff_ns;  // cap of the sync-free polling backoff (0 = spin)
  int* derr;            // device copy of the watchdog word: later polls give up at once
  uint32_t wd_spins;    // unsuccessful polls before the watchdog trips (kWatchdogSpins)
  unsigned long long* sf_trace;  // SPTRSV_SF_TRACE builds: {claim, done} globaltimer per row
};

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#ifdef SPTRSV_SF_TRACE
#define SF_TRACE(st, row, which) \
  do {                                                       \
    if ((st).sf_trace) (st).sf_trace[2 * (size_t)(row) + (which)] = gtimer(); \
  } while (0)
#else
#define SF_TRACE(st, row, which) \
  do {                         \
  } while (0)
#endif

__device__ __forceinline__ void reset_tickets(const SolveState& st, int tid, int nthreads) {
  for (int t = tid; t < st.nticket; t += nthreads) st.tickets[t] = 0;
}

// permute-in, block 0, thread 0: hand out this solve's epochs [base, base + span)
__device__ __forceinline__ void advance_epoch(const SolveState& st) {
  if (st.span && st.epoch_dev) {
    const uint32_t base = st.epoch_dev[1] + 1u;
    st.epoch_dev[0] = base;
    st.epoch_dev[1] = base + st.span - 1u;
  }
}

// this launch's epoch (written by permute-in, an earlier kernel of the stream)
__device__ __forceinline__ uint32_t solve_epoch(const SolveState& st) {
  return *(volatile const uint32_t*)st.epoch_dev + st.epoch_off;
}

__device__ __forceinline__ void watchdog_trip(const SolveState& st) {
  if (st.error) *(volatile int*)st.error = 1;
  if (st.derr) *(volatile int*)st.derr = 1;
}

// One more unsuccessful poll: true = give up (this poll's watchdog tripped,
// or another one already did -- checked every 1024 polls, so the chunk
// launches after a trip do not each spin kWatchdogSpins again).  The lanes'
// counters can differ (per-lane loops), so a loop whose condition is a
// full-warp vote takes the decision with __any_sync: a lane that left such a
// loop alone would leave the others blocked in the next vote.
__device__ __forceinline__ bool wd_giveup(uint32_t& spins, const SolveState& st) {
  if (++spins > st.wd_spins) {
    watchdog_trip(st);
    return true;
  }
  return (spins & 1023u) == 0 && st.derr && *(volatile int*)st.derr;
}

// ------------------------------------------------------------------ permute
// bw[k] = b[perm[k]] / d_k (as * rd), xs[k] = SENT (if a sync-free triangle
// polls it).  nrhs == 1; stride = ldb for row-major input, 1 otherwise.
template <typename T>
__global__ void perm_in_1(int n, const int* __restrict__ perm, const T* __restrict__ rd, const T* __restrict__ b,
                          int64_t stride, T* __restrict__ bw, T* __restrict__ xs, int fill_sent, SolveState st,
                          T* __restrict__ part, int npart) {
  if (blockIdx.x == 0) {
    reset_tickets(st, threadIdx.x, blockDim.x);
    if (threadIdx.x == 0) advance_epoch(st);
  }
  int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k < n) {
    bw[k] = b[(int64_t)perm[k] * stride] * rd[k];
    if (fill_sent) xs[k] = sent<T>();
  }
  if (k < npart) part[k] = sent<T>();  // split long rows' partial sums (tri_sf_items)
}

// x[perm[k]] = xs[k]
template <typename T>
__global__ void perm_out_1(int n, const int* __restrict__ perm, const T* __restrict__ xs, T* __restrict__ x,
                           int64_t stride) {
  int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k < n) x[(int64_t)perm[k] * stride] = xs[k];
}

// Column-major B (n x nrhs, ldb) -> row-major bw.  A block owns 32 original
// rows i and walks ALL the RHS columns in 32 x 32 tiles transposed through
// shared memory: reads are coalesced along i (256 B per column), writes are
// 256 B pieces of the permuted rows iperm[i], and each 4 KB (512-RHS) row is
// completed by one block within a few microseconds (DRAM-page friendly, no
// partial sectors left in L2).  The next tile's loads are in flight while
// the current tile is stored.
template <typename T>
__global__ void __launch_bounds__(256) perm_in_cm(int n, int nrhs, const int* __restrict__ iperm,
                                                  const T* __restrict__ rd, const T* __restrict__ b, int64_t ldb,
                                                  T* __restrict__ bw, T* __restrict__ xs, int fill_sent,
                                                  SolveState st) {
  __shared__ T tile[32][33];
  __shared__ int ks[32];
  __shared__ T rs[32];
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
  if (blockIdx.x == 0) {
    reset_tickets(st, threadIdx.x, 256);
    if (threadIdx.x == 0) advance_epoch(st);
  }
  const int i0 = blockIdx.x * 32, i = i0 + tx;
  const bool iv = i < n;
  if (threadIdx.x < 32) {
    const int k = iv ? iperm[i] : 0;
    ks[tx] = k;
    rs[tx] = iv ? rd[k] : T(0);
  }
  T v[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const int c = ty + 8 * j;
    v[j] = (iv && c < nrhs) ? ldg_nc(b + i + (int64_t)c * ldb) : T(0);
  }
  for (int c0 = 0; c0 < nrhs; c0 += 32) {
    __syncthreads();  // the previous tile has been read out
#pragma unroll
    for (int j = 0; j < 4; ++j) tile[ty + 8 * j][tx] = v[j];
    __syncthreads();
    if (c0 + 32 < nrhs) {
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int c = c0 + 32 + ty + 8 * j;
        v[j] = (iv && c < nrhs) ? ldg_nc(b + i + (int64_t)c * ldb) : T(0);
      }
    }
    const int c = c0 + tx;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int ii = ty + 8 * j;
      if (i0 + ii < n && c < nrhs) {
        const int64_t o = (int64_t)ks[ii] * nrhs + c;
        bw[o] = tile[tx][ii] * rs[ii];
        if (fill_sent) xs[o] = sent<T>();
      }
    }
  }
}

// x = P^T xs for column-major X: the mirror of perm_in_cm (a block gathers
// 256 B pieces of 32 permuted rows, writes 32 consecutive rows per column).
template <typename T>
__global__ void __launch_bounds__(256) perm_out_cm(int n, int nrhs, const int* __restrict__ iperm,
                                                   const T* __restrict__ xs, T* __restrict__ x, int64_t ldx) {
  __shared__ T tile[32][33];
  __shared__ int ks[32];
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
  const int i0 = blockIdx.x * 32;
  if (threadIdx.x < 32) ks[tx] = i0 + tx < n ? iperm[i0 + tx] : 0;
  __syncthreads();
  T v[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const int ii = ty + 8 * j;
    v[j] = (i0 + ii < n && tx < nrhs) ? ldg_nc(xs + (int64_t)ks[ii] * nrhs + tx) : T(0);
  }
  const int i = i0 + tx;
  for (int c0 = 0; c0 < nrhs; c0 += 32) {
    __syncthreads();
#pragma unroll
    for (int j = 0; j < 4; ++j) tile[ty + 8 * j][tx] = v[j];
    __syncthreads();
    if (c0 + 32 < nrhs) {
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int ii = ty + 8 * j, c = c0 + 32 + tx;
        v[j] = (i0 + ii < n && c < nrhs) ? ldg_nc(xs + (int64_t)ks[ii] * nrhs + c) : T(0);
      }
    }
    if (i < n) {
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int c = c0 + ty + 8 * j;
        if (c < nrhs) x[i + (int64_t)c * ldx] = tile[tx][ty + 8 * j];
      }
    }
  }
}

// Row-major B (ldb >= nrhs): bw[k*nrhs + c] = b[perm[k]*ldb + c] * rd[k]
template <typename T>
__global__ void perm_in_rm(int n, int nrhs, const int* __restrict__ perm, const T* __restrict__ rd,
                           const T* __restrict__ b, int64_t ldb, T* __restrict__ bw, T* __restrict__ xs,
                           int fill_sent, SolveState st) {
  if (blockIdx.x == 0) {
    reset_tickets(st, threadIdx.x, blockDim.x);
    if (threadIdx.x == 0) advance_epoch(st);
  }
  int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e < (int64_t)n * nrhs) {
    int k = (int)(e / nrhs), c = (int)(e % nrhs);
    bw[e] = b[(int64_t)perm[k] * ldb + c] * rd[k];
    if (fill_sent) xs[e] = sent<T>();
  }
}

template <typename T>
__global__ void perm_out_rm(int n, int nrhs, const int* __restrict__ perm, const T* __restrict__ xs,
                            T* __restrict__ x, int64_t ldx) {
  int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e < (int64_t)n * nrhs) {
    int k = (int)(e / nrhs), c = (int)(e % nrhs);
    x[(int64_t)perm[k] * ldx + c] = xs[e];
  }
}

// ------------------------------------------------------- K1: diagonal triangle
// SPTRSV-COMPLETELYPARALLEL (L247 structure 1, Alg 7): x_i = b_i / d_i;
// the 1/d_i scaling already happened in permute-in, so this is x = bw.
template <typename T>
__global__ void tri_diag(int r0, int m, int nrhs, const T* __restrict__ bw, T* __restrict__ xs) {
  int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e < (int64_t)m * nrhs) xs[(int64_t)r0 * nrhs + e] = bw[(int64_t)r0 * nrhs + e];
}

// ------------------------------------------ square blocks: b_rows -= A x_cols
// SPMV-SCALAR-CSR / -DCSR (L249-L250, Alg 7): one thread per row.
template <typename T, bool DCSR>
__global__ void sq_scalar_1(int nzr, int r0, const int* __restrict__ rows, const int* __restrict__ rp,
                            const int* __restrict__ ci, const T* __restrict__ val, const T* __restrict__ xs,
                            T* __restrict__ bw) {
  int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= nzr) return;
  int r = DCSR ? rows[t] : r0 + t;
  int a = rp[t], e = rp[t + 1];
  T s = 0;
  for (int p = a; p < e; ++p) s += ldg_nc(val + p) * ldg_nc(xs + ldg_nc(ci + p));
  bw[r] -= s;
}

// SPMV-VECTOR-CSR / -DCSR (L249-L250, Alg 7): a warp per row.
template <typename T, bool DCSR>
__global__ void sq_vector_1(int nzr, int r0, const int* __restrict__ rows, const int* __restrict__ rp,
                            const int* __restrict__ ci, const T* __restrict__ val, const T* __restrict__ xs,
                            T* __restrict__ bw) {
  int wid = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (wid >= nzr) return;
  int a = rp[wid], e = rp[wid + 1];
  T s = 0;
  for (int p = a + lane; p < e; p += 32) s += ldg_nc(val + p) * ldg_nc(xs + ldg_nc(ci + p));
  s = warp_sum(s);
  if (lane == 0) {
    int r = DCSR ? rows[wid] : r0 + wid;
    bw[r] -= s;
  }
}

// B200 square update (nrhs == 1, selector B200): nnz-balanced ROW BLOCKS.
// The upload cuts the stored rows into work items of <= 32 consecutive rows
// holding <= kSqNB entries together (a row longer than kSqNB is an item of
// its own, cut into kSqLW-entry chunks when longer still), one warp each.
// A block streams its entries coalesced -- every lane issues all its
// (ci, val) loads, then all its x gathers, before the first use, so
// kSqNB / 32 independent gathers per lane are in flight -- into shared
// memory as products; then lane t sums row t0 + t from shared memory and
// updates b'.  Rows of any length mix in one launch with full lanes (the
// paper's scalar / vector kernels leave lanes idle on short rows and
// serialise long ones, L249-L250).  A row cut into several chunks adds its
// partial sums with atomics (summation order then varies, reading R22).
#ifndef SPTRSV_SQ_NB
#define SPTRSV_SQ_NB 256  // entries per row block (tuning builds may change it)
#endif
constexpr int kSqNB = SPTRSV_SQ_NB, kSqLW = 1024;
struct SqItem {
  int t0, t1;  // stored rows [t0, t1); bit 31 of t1: chunk of a split row (atomic update)
  int p0, p1;  // entries [p0, p1)
};

template <typename T, bool DCSR>
__global__ void __launch_bounds__(256) sq_adapt_1(int nitem, int r0, const SqItem* __restrict__ items,
                                                  const int* __restrict__ rows, const int* __restrict__ rp,
                                                  const int* __restrict__ ci, const T* __restrict__ val,
                                                  const T* __restrict__ xs, T* __restrict__ bw) {
  // One item per warp.  Every load that does not depend on x (entries, row
  // bounds, DCSR row ids, the b' values) is issued together with the entry
  // loads, so the item's dependent chain is header -> entries -> x gathers.
  // (A persistent grid with next-item prefetch measured slower on C3.)
  __shared__ T prod[8][kSqNB];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int w = blockIdx.x * 8 + warp;
  if (w >= nitem) return;
  const int4 it = __ldg((const int4*)(items + w));
  const int t0 = it.x, t1 = it.y & 0x7fffffff, a = it.z, e = it.w;
  if (it.y < 0 || e - a > kSqNB) {  // one long row, or a chunk of a split one (any length)
    T s[4] = {0, 0, 0, 0};
    for (int p = a + lane; p < e; p += 128) {
      int j[4];
      T v[4], x[4];
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (p + 32 * u < e) {
          j[u] = ldg_nc(ci + p + 32 * u);
          v[u] = ldg_nc(val + p + 32 * u);
        }
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (p + 32 * u < e) x[u] = ldg_nc(xs + j[u]);
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (p + 32 * u < e) s[u] += v[u] * x[u];
    }
    const T sum = warp_sum((s[0] + s[1]) + (s[2] + s[3]));
    if (lane == 0) {
      const int r = DCSR ? rows[t0] : r0 + t0;
      if (it.y < 0)
        atomicAdd(bw + r, -sum);
      else
        bw[r] -= sum;
    }
    return;
  }
  T* pr = prod[warp];
  int j[kSqNB / 32];
  T v[kSqNB / 32], x[kSqNB / 32];
#pragma unroll
  for (int u = 0; u < kSqNB / 32; ++u) {
    const int p = a + 32 * u + lane;
    if (p < e) {
      j[u] = ldg_nc(ci + p);
      v[u] = ldg_nc(val + p);
    }
  }
  const int t = t0 + lane;
  int q0 = 0, q1 = 0, r = 0;
  T br = T(0);
  if (t < t1) {
    q0 = __ldg(rp + t) - a;
    q1 = __ldg(rp + t + 1) - a;
    r = DCSR ? __ldg(rows + t) : r0 + t;
    if (q1 > q0) br = bw[r];  // this item is the only writer of row r
  }
#pragma unroll
  for (int u = 0; u < kSqNB / 32; ++u)
    if (a + 32 * u + lane < e) x[u] = ldg_nc(xs + j[u]);
#pragma unroll
  for (int u = 0; u < kSqNB / 32; ++u)
    if (a + 32 * u + lane < e) pr[32 * u + lane] = v[u] * x[u];
  __syncwarp();
  if (q1 > q0) {
    T sum = 0;
    for (int q = q0; q < q1; ++q) sum += pr[q];
    bw[r] = br - sum;
  }
}

// SpMM update for nrhs > 1 (K9): a group of G lanes per row, lanes over the
// RHS columns (RPT per lane per pass), entries of the row two at a time so
// 2*RPT independent X gathers per lane are in flight (round-1 ncu: one entry
// at a time left the kernel latency-bound at 3.5 TB/s, long_scoreboard 116).
template <typename T, bool NC>
__device__ __forceinline__ T ldx(const T* p) {
  if constexpr (NC) return ldg_nc(p);
  else return *p;
}

template <typename T, int RPT, bool NC = true, int UN = 1>
__device__ __forceinline__ void gather_row_update(T (&acc)[RPT], int a, int e, const int* __restrict__ ci,
                                                  const T* __restrict__ val, const T* __restrict__ xs, int nrhs,
                                                  int cbase, int G, int ncol) {
  int p = a;
  if constexpr (UN == 2) {
    for (; p + 1 < e; p += 2) {
      const int j0 = ldg_nc(ci + p), j1 = ldg_nc(ci + p + 1);
      const T v0 = ldg_nc(val + p), v1 = ldg_nc(val + p + 1);
      const T* x0 = xs + (int64_t)j0 * nrhs + cbase;
      const T* x1 = xs + (int64_t)j1 * nrhs + cbase;
      T y0[RPT], y1[RPT];
#pragma unroll
      for (int t = 0; t < RPT; ++t)
        if (G * t < ncol) {
          y0[t] = ldx<T, NC>(x0 + G * t);
          y1[t] = ldx<T, NC>(x1 + G * t);
        }
#pragma unroll
      for (int t = 0; t < RPT; ++t)
        if (G * t < ncol) acc[t] += v0 * y0[t] + v1 * y1[t];
    }
  }
  for (; p < e; ++p) {
    const int j0 = ldg_nc(ci + p);
    const T v0 = ldg_nc(val + p);
    const T* x0 = xs + (int64_t)j0 * nrhs + cbase;
#pragma unroll
    for (int t = 0; t < RPT; ++t)
      if (G * t < ncol) acc[t] += v0 * ldx<T, NC>(x0 + G * t);
  }
}

template <typename T, int G, int RPT, int UN, bool DCSR>
__global__ void sq_multi(int nzr, int r0, const int* __restrict__ rows, const int* __restrict__ rp,
                         const int* __restrict__ ci, const T* __restrict__ val, const T* __restrict__ xs,
                         T* __restrict__ bw, int nrhs) {
  int g = (blockIdx.x * blockDim.x + threadIdx.x) / G, lane = threadIdx.x % G;
  if (g >= nzr) return;
  int r = DCSR ? rows[g] : r0 + g;
  int a = rp[g], e = rp[g + 1];
  for (int c0 = 0; c0 < nrhs; c0 += G * RPT) {
    T acc[RPT];
#pragma unroll
    for (int t = 0; t < RPT; ++t) acc[t] = 0;
    // columns c0 + lane + G*t < nrhs  <=>  G*t < nrhs - c0 - lane
    gather_row_update<T, RPT, true, UN>(acc, a, e, ci, val, xs, nrhs, c0 + lane, G, nrhs - c0 - lane);
    T* br = bw + (int64_t)r * nrhs + c0 + lane;
#pragma unroll
    for (int t = 0; t < RPT; ++t)
      if (c0 + lane + G * t < nrhs) br[G * t] -= acc[t];
  }
}

// SpMM square update with RHS TILING (B200, nrhs > 1): blockIdx.y selects a
// tile of G*RPT right-hand-side columns and the grid is scheduled tile-major
// (x fastest), so all resident CTAs gather from the same column tile of X:
// the tile's rows of X (cols x G*RPT x 8 B) stay L2-resident instead of every
// gather of a 4 KB X row missing L2 (round 1: 2.66x the algorithmic DRAM
// bytes on C5's largest square).  The matrix is re-streamed once per tile.
template <typename T, int G, int RPT, int UN, bool DCSR>
__global__ void sq_multi_tiled(int nzr, int r0, const int* __restrict__ rows, const int* __restrict__ rp,
                               const int* __restrict__ ci, const T* __restrict__ val, const T* __restrict__ xs,
                               T* __restrict__ bw, int nrhs) {
  const int c0 = blockIdx.y * (G * RPT);
  const int g = (blockIdx.x * blockDim.x + threadIdx.x) / G, lane = threadIdx.x % G;
  if (g >= nzr) return;
  const int r = DCSR ? rows[g] : r0 + g;
  const int a = rp[g], e = rp[g + 1];
  if (a == e) return;
  T acc[RPT];
#pragma unroll
  for (int t = 0; t < RPT; ++t) acc[t] = 0;
  gather_row_update<T, RPT, true, UN>(acc, a, e, ci, val, xs, nrhs, c0 + lane, G, nrhs - c0 - lane);
  T* br = bw + (int64_t)r * nrhs + c0 + lane;
#pragma unroll
  for (int t = 0; t < RPT; ++t)
    if (c0 + lane + G * t < nrhs) br[G * t] -= acc[t];
}

// ------------------------------------------------- K2: one level of a triangle
// SPTRSV-LEVEL-SET (Alg 2 L88-L98; L247 "a thread or a 32-thread warp"): after
// the level reorder every level is a contiguous row range [ra, rb).  One
// launch per level; the launch boundary is the barrier of Alg 2 L96.
template <typename T, bool WARP>
__global__ void tri_level_1(int ra, int rb, int r0, const int* __restrict__ rp, const int* __restrict__ ci,
                            const T* __restrict__ val, const T* __restrict__ bw, T* __restrict__ xs) {
  int lane = threadIdx.x & 31;
  int r = WARP ? ra + ((blockIdx.x * blockDim.x + threadIdx.x) >> 5) : ra + blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= rb) return;
  int a = rp[r - r0], e = rp[r - r0 + 1];
  T s = 0;
  if (WARP) {
    for (int p = a + lane; p < e; p += 32) s += ldg_nc(val + p) * xs[ldg_nc(ci + p)];
    s = warp_sum(s);
    if (lane == 0) xs[r] = bw[r] - s;
  } else {
    for (int p = a; p < e; ++p) s += ldg_nc(val + p) * xs[ldg_nc(ci + p)];
    xs[r] = bw[r] - s;
  }
}

// x_r = b'_r - sum_j l'_rj x_j for the RHS columns this lane owns.  NC:
// the x_j come from earlier launches (level-set) and may use the
// non-coherent path; the single-CTA chain reads them with plain loads.
template <typename T, int G, int RPT, bool NC, int UN>
__device__ __forceinline__ void row_multi_solve(int r, int a, int e, const int* __restrict__ ci,
                                                const T* __restrict__ val, const T* __restrict__ bw,
                                                T* __restrict__ xs, int nrhs, int lane) {
  for (int c0 = 0; c0 < nrhs; c0 += G * RPT) {
    T acc[RPT];
#pragma unroll
    for (int t = 0; t < RPT; ++t) acc[t] = 0;
    gather_row_update<T, RPT, NC, UN>(acc, a, e, ci, val, xs, nrhs, c0 + lane, G, nrhs - c0 - lane);
    T* xo = xs + (int64_t)r * nrhs + c0 + lane;
    const T* bo = bw + (int64_t)r * nrhs + c0 + lane;
#pragma unroll
    for (int t = 0; t < RPT; ++t)
      if (c0 + lane + G * t < nrhs) xo[G * t] = bo[G * t] - acc[t];
  }
}

template <typename T, int G, int RPT, int UN>
__global__ void tri_level_multi(int ra, int rb, int r0, const int* __restrict__ rp, const int* __restrict__ ci,
                                const T* __restrict__ val, const T* __restrict__ bw, T* __restrict__ xs,
                                int nrhs) {
  int r = ra + (blockIdx.x * blockDim.x + threadIdx.x) / G, lane = threadIdx.x % G;
  if (r >= rb) return;
  row_multi_solve<T, G, RPT, true, UN>(r, rp[r - r0], rp[r - r0 + 1], ci, val, bw, xs, nrhs, lane);
}

// ---------------------------------------- K4: single-CTA level chain (unstaged)
// One CTA walks the levels in order and separates them with bar.sync (tens of
// cycles) instead of a kernel launch or cross-SM flags.  Rows solved in
// earlier levels are read with plain loads, which are coherent inside the SM
// after bar.sync -- NOT through the non-coherent (ld.global.nc) path.
// Used for nrhs > 1 and for rows longer than the staged kernel's stage.
template <typename T, bool WARP>
__global__ void __launch_bounds__(1024) tri_chain_1(int r0, int nlev, const int* __restrict__ lp,
                                                    const int* __restrict__ rp, const int* __restrict__ ci,
                                                    const T* __restrict__ val, const T* __restrict__ bw,
                                                    T* __restrict__ xs) {
  const int tid = threadIdx.x, nt = blockDim.x;
  const int lane = tid & 31, wid = tid >> 5, nw = nt >> 5;
  for (int l = 0; l < nlev; ++l) {
    int ra = r0 + lp[l], rb = r0 + lp[l + 1];
    if (WARP) {
      for (int r = ra + wid; r < rb; r += nw) {
        int a = rp[r - r0], e = rp[r - r0 + 1];
        T s = 0;
        for (int p = a + lane; p < e; p += 32) s += ldg_nc(val + p) * xs[ldg_nc(ci + p)];
        s = warp_sum(s);
        if (lane == 0) xs[r] = bw[r] - s;
      }
    } else {
      for (int r = ra + tid; r < rb; r += nt) {
        int a = rp[r - r0], e = rp[r - r0 + 1];
        T s = bw[r];
        for (int p = a; p < e; ++p) s -= ldg_nc(val + p) * xs[ldg_nc(ci + p)];
        xs[r] = s;
      }
    }
    __syncthreads();
  }
}

template <typename T, int G, int RPT, int UN>
__global__ void __launch_bounds__(1024) tri_chain_multi(int r0, int nlev, const int* __restrict__ lp,
                                                        const int* __restrict__ rp, const int* __restrict__ ci,
                                                        const T* __restrict__ val, const T* __restrict__ bw,
                                                        T* __restrict__ xs, int nrhs) {
  const int grp = threadIdx.x / G, ng = blockDim.x / G, lane = threadIdx.x % G;
  for (int l = 0; l < nlev; ++l) {
    int ra = r0 + lp[l], rb = r0 + lp[l + 1];
    for (int r = ra + grp; r < rb; r += ng)
      row_multi_solve<T, G, RPT, false, UN>(r, rp[r - r0], rp[r - r0 + 1], ci, val, bw, xs, nrhs, lane);
    __syncthreads();
  }
}

// ------------------------------------------------ K3: sync-free (multi-CTA)
// Sync-free SpTRSV (Alg 3) for sm_100a in its pull (CSR) form.
// Components are claimed from a per-segment ticket in row order, so every
// dependency of a claimed row was claimed earlier by a running warp: no
// deadlock whatever the CTA scheduling.  A dependency is "satisfied" (the
// in-degree test of Alg 3) when its x_j is no longer the sentinel
// (nrhs == 1) or its row flag carries this solve's epoch (nrhs > 1).
//
// Polling discipline: in the thread-per-row and multi-RHS kernels a warp
// whose polls made no progress sleeps (__nanosleep, exponential backoff
// capped at SolveState::backoff_ns, SPTRSV_SF_BACKOFF) before polling again,
// so blocked warps do not saturate the LSU / L2 with strong loads (round-1
// ncu: the un-throttled kernel ran L1TEX at 95% with lg_throttle the second
// stall reason, profiles/r01_c3_v0_ncu.md).  The warp-per-row kernel spins
// (measured faster on C3/C4: its warps poll few, long rows).  The resident
// grid is also sized to ~2 levels of rows (exec.cu), so few warps spin.
constexpr unsigned kBackoffMinNs = 32;

__device__ __forceinline__ unsigned backoff(unsigned ns, unsigned max_ns) {
  if (max_ns == 0) return 0;  // pure spinning
  ns = ns ? min(ns * 2u, max_ns) : min(kBackoffMinNs, max_ns);
  __nanosleep(ns);
  return ns;
}

__device__ __forceinline__ uint32_t ld_flag(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_flag(uint32_t* p, uint32_t v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// Thread-per-component with warp help for long rows: a warp claims 32
// consecutive rows.  A row with <= LONG dependencies is solved by its own
// lane, which consumes its dependencies in batches of U independent loads,
// stopping at the first unsolved one and retrying on the next pass
// (non-blocking, so a lane never blocks a lower lane of its own warp that it
// depends on).  A longer row (the power-law hubs of L136, which serialise a
// lane for thousands of cycles) is solved by the WHOLE warp, 32*U entries per
// attempt, lowest such row first; an attempt that meets an unsolved
// dependency is abandoned without side effects and retried after the next
// thread pass, so rows of the same chunk that the long row waits for keep
// progressing (no deadlock: the long row only waits on lower rows, and the
// lower long rows are finished first).
template <typename T, int U, int LONG>
__global__ void __launch_bounds__(256) tri_syncfree_thread(int r0, int m, const int* __restrict__ rp,
                                                           const int* __restrict__ ci, const T* __restrict__ val,
                                                           const T* __restrict__ bw, T* __restrict__ xs,
                                                           SolveState st, int slot) {
  const int lane = threadIdx.x & 31;
  uint32_t* ticket = st.tickets + slot;
  while (true) {
    int base = 0;
    if (lane == 0) base = (int)atomicAdd(ticket, 32u);
    base = __shfl_sync(0xffffffffu, base, 0);
    if (base >= m) break;
    const int k = base + lane;
    bool done = k >= m;
    const int r = r0 + k;
    int p = 0, e = 0;
    T s = 0;
    if (!done) {
      SF_TRACE(st, r, 0);
      p = rp[k];
      e = rp[k + 1];
      s = bw[r];
    }
    const bool islong = !done && e - p > LONG;
    uint32_t spins = 0;
    unsigned ns = 0;
    while (__any_sync(0xffffffffu, !done)) {
      bool prog = false;
      if (!done && !islong) {
        bool progress = true;
        while (p < e && progress) {
          const int cnt = min(U, e - p);
          int j[U];
          T v[U], x[U];
#pragma unroll
          for (int u = 0; u < U; ++u)
            if (u < cnt) {
              j[u] = ldg_nc(ci + p + u);
              v[u] = ldg_nc(val + p + u);
            }
#pragma unroll
          for (int u = 0; u < U; ++u)
            if (u < cnt) x[u] = ld_strong(xs + j[u]);
          int took = 0;
#pragma unroll
          for (int u = 0; u < U; ++u)
            if (u < cnt && took == u && !is_sent(x[u])) {
              s -= v[u] * x[u];
              ++took;
            }
          p += took;
          prog |= took > 0;
          progress = took == cnt;
        }
        if (p == e) {
          st_strong(xs + r, s);
          SF_TRACE(st, r, 1);
          done = true;
          prog = true;
        }
      }
      // warp pass: the lowest pending long row, 32*U entries per attempt
      const unsigned lm = __ballot_sync(0xffffffffu, !done && islong);
      if (lm) {
        const int ow = __ffs(lm) - 1;
        int wp = __shfl_sync(0xffffffffu, p, ow);
        const int we = __shfl_sync(0xffffffffu, e, ow);
        T acc = 0;
        while (wp < we) {
          int j[U];
          T v[U], x[U];
          bool ready = true;
#pragma unroll
          for (int u = 0; u < U; ++u) {
            const int q = wp + lane + 32 * u;
            if (q < we) {
              j[u] = ldg_nc(ci + q);
              v[u] = ldg_nc(val + q);
            }
          }
#pragma unroll
          for (int u = 0; u < U; ++u)
            if (wp + lane + 32 * u < we) {
              x[u] = ld_strong(xs + j[u]);
              ready &= !is_sent(x[u]);
            }
          if (!__all_sync(0xffffffffu, ready)) break;  // abandon; retry after the next thread pass
#pragma unroll
          for (int u = 0; u < U; ++u)
            if (wp + lane + 32 * u < we) acc += v[u] * x[u];
          wp += 32 * U;
          prog = true;
        }
        acc = warp_sum(acc);
        if (lane == ow) {
          s -= acc;
          p = min(wp, we);
          if (p == e) {
            st_strong(xs + r, s);
            SF_TRACE(st, r, 1);
            done = true;
          }
        }
      }
      if (!__any_sync(0xffffffffu, prog)) {
        if (wd_giveup(spins, st)) {
          done = true;  // give up: garbage result, reported to the host
        } else {
          ns = backoff(ns, st.backoff_ns);
        }
      } else {
        ns = 0;
      }
    }
  }
}

// Warp-per-component (long rows): lanes stride the dependencies, U per lane
// per round (32*U entries: every column index and value of the round is
// loaded BEFORE the first poll, so the matrix stream never sits behind a
// dependency wait); a lane spins only on dependencies, which all precede the
// row in ticket order.
template <typename T, int U>
__global__ void __launch_bounds__(256) tri_syncfree_warp(int r0, int m, const int* __restrict__ rp,
                                                         const int* __restrict__ ci, const T* __restrict__ val,
                                                         const T* __restrict__ bw, T* __restrict__ xs,
                                                         SolveState st, int slot) {
  const int lane = threadIdx.x & 31;
  uint32_t* ticket = st.tickets + slot;
  while (true) {
    int k = 0;
    if (lane == 0) k = (int)atomicAdd(ticket, 1u);
    k = __shfl_sync(0xffffffffu, k, 0);
    if (k >= m) break;
    const int r = r0 + k;
    if (lane == 0) SF_TRACE(st, r, 0);
    const int a = rp[k], e = rp[k + 1];
    T s = 0;
    for (int p0 = a; p0 < e; p0 += 32 * U) {
      int j[U];
      T v[U], x[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        int p = p0 + lane + 32 * u;
        if (p < e) {
          j[u] = ldg_nc(ci + p);
          v[u] = ldg_nc(val + p);
        }
      }
#pragma unroll
      for (int u = 0; u < U; ++u)
        if (p0 + lane + 32 * u < e) x[u] = ld_strong(xs + j[u]);
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (p0 + lane + 32 * u < e) {
          uint32_t spins = 0;
          while (is_sent(x[u])) {
            if (wd_giveup(spins, st)) break;
            x[u] = ld_strong(xs + j[u]);
          }
          s += v[u] * x[u];
        }
      }
    }
    s = warp_sum(s);
    if (lane == 0) {
      st_strong(xs + r, bw[r] - s);
      SF_TRACE(st, r, 1);
    }
  }
}

// Sync-free over nnz-balanced ROW BLOCKS (B200 selector, nrhs == 1): the
// sync-free solve of Alg 3 (L105-L125) in pull form, with the work cut at
// upload into items of <= 32 consecutive rows holding <= kSfNB off-diagonal
// entries together (exec.cu build_sf_items); a row longer than kSfNB is cut
// into kSfNB-entry PIECES, each an item of its own:
//   - a partial piece (kind 1) writes its partial sum to a slot of `part`
//     (value-as-flag: slots hold the sentinel until written, reset by
//     permute-in);
//   - the row's last piece (kind 2) adds its own entries and the partial sums
//     of the earlier pieces, in piece order (deterministic), and publishes x.
// A warp claims one item per ticket (row order: deadlock-free like K3, the
// pieces of a row precede its last piece).  All entries of the item are
// loaded coalesced and all their x_j polled at once (kSfNB/32 loads in flight
// per lane); a ready product goes to shared memory and bumps its row's
// counter; a row whose counter is complete is summed by its own lane in entry
// order and published with one strong store.  Dependencies inside the item
// are read from shared memory (the rows' solved x are forwarded there), so a
// chain inside an item costs no L2 round trip.  Long rows (the power-law hubs
// of L136) thus take one round of loads spread over several warps instead of
// a serial walk by one warp.
#ifndef SPTRSV_SF_NB
#define SPTRSV_SF_NB 256
#endif
#ifndef SPTRSV_SF_MINB
#define SPTRSV_SF_MINB 2  // resident CTAs per SM requested from ptxas
#endif
constexpr int kSfNB = SPTRSV_SF_NB;
#ifndef SPTRSV_SF_LONG
#define SPTRSV_SF_LONG 64  // round-2 sweep on C3 (16 / 32 / 64 / 96 / 128): 3.48 / 3.10 / 2.95 / 2.95 / 2.97 ms
#endif
constexpr int kSfLong = SPTRSV_SF_LONG;  // tri_sf_mixed: rows with more entries get a warp
#ifndef SPTRSV_SF_U
#define SPTRSV_SF_U 4  // tri_sf_mixed: loads a lane of a row group issues per batch
#endif
#ifndef SPTRSV_SF_POLLS
#define SPTRSV_SF_POLLS 1
#endif
#ifndef SPTRSV_SF_GAP
#define SPTRSV_SF_GAP 64
#endif
constexpr int kSfPolls = SPTRSV_SF_POLLS, kSfGap = SPTRSV_SF_GAP;  // tri_sf_mixed: staggered polls
#ifndef SPTRSV_SF_WU
#define SPTRSV_SF_WU 4
#endif
constexpr int kSfWU = SPTRSV_SF_WU, kSfW = 32 * kSfWU;  // tri_sf_wrow: entries per item
struct SfItem {
  int t0, t1;  // local rows [t0, t1) (a piece: t1 = t0 + 1)
  int p0, p1;  // entries [p0, p1) of the segment's CSR
  int kind;    // 0 rows, 1 partial piece (-> part[s0]), 2 last piece (+ part[s0 .. s1))
  int s0, s1, pad;
};

template <typename T>
__global__ void __launch_bounds__(256, SPTRSV_SF_MINB) tri_sf_items(int r0, int nitem, const SfItem* __restrict__ items,
                                                    const int* __restrict__ rp, const int* __restrict__ ci,
                                                    const T* __restrict__ val, const T* __restrict__ bw,
                                                    T* __restrict__ xs, T* __restrict__ part, SolveState st,
                                                    int slot) {
  constexpr int U = kSfNB / 32;
  __shared__ T prod_s[8][kSfNB];
  __shared__ T xloc_s[8][32];
  __shared__ int lrp_s[8][33];
  __shared__ int cnt_s[8][32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  T* prod = prod_s[warp];
  T* xloc = xloc_s[warp];
  int* lrp = lrp_s[warp];
  int* cnt = cnt_s[warp];
  uint32_t* ticket = st.tickets + slot;
  for (;;) {
    int w = 0;
    if (lane == 0) w = (int)atomicAdd(ticket, 1u);
    w = __shfl_sync(0xffffffffu, w, 0);
    if (w >= nitem) break;
    const int4 h0 = __ldg((const int4*)(items + w));
    const int4 h1 = __ldg((const int4*)(items + w) + 1);
    const int t0 = h0.x, nr = h0.y - h0.x, p0 = h0.z, ne = h0.w - h0.z, kind = h1.x;
    // row pointers of the item, relative to p0 (a piece is one row of ne entries)
    if (lane < nr) {
      lrp[lane] = kind == 0 ? rp[t0 + lane] - p0 : 0;
      SF_TRACE(st, r0 + t0 + lane, 0);
    }
    if (lane == 0) lrp[nr] = ne;
    cnt[lane] = 0;
    xloc[lane] = sent<T>();
    __syncwarp();
    const int jlo = r0 + t0, jhi = r0 + t0 + nr;  // the item's own rows (global)
    const T bwr = (lane < nr && kind != 1) ? bw[jlo + lane] : T(0);  // off the critical path
    int j[U], rw[U];
    T v[U], x[U];
    uint32_t pend = 0;
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int e = lane + 32 * u;
      if (e < ne) {
        j[u] = ldg_nc(ci + p0 + e);
        v[u] = ldg_nc(val + p0 + e);
        pend |= 1u << u;
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {  // row of entry e: the last row start <= e
      const int e = lane + 32 * u;
      int lo = 0;
      if (e < ne && kind == 0) {
        int hi = nr;  // lrp[lo] <= e < lrp[hi]
        while (hi - lo > 1) {
          const int mid = (lo + hi) >> 1;
          if (lrp[mid] <= e) lo = mid;
          else hi = mid;
        }
      }
      rw[u] = lo;
    }
    bool rdone = lane >= nr;  // this lane's row (lane < nr) is published
    uint32_t spins = 0;
    unsigned ns = 0;
    for (;;) {
      // poll every pending dependency at once (shared memory for the item's own rows)
#pragma unroll
      for (int u = 0; u < U; ++u)
        if (pend & (1u << u)) {
          if (kind == 0 && j[u] >= jlo && j[u] < jhi)
            x[u] = *(volatile T*)&xloc[j[u] - jlo];
          else
            x[u] = ld_strong(xs + j[u]);
        }
      bool prog = false;
#pragma unroll
      for (int u = 0; u < U; ++u)
        if ((pend & (1u << u)) && !is_sent(x[u])) {
          prod[lane + 32 * u] = v[u] * x[u];
          atomicAdd(&cnt[rw[u]], 1);
          pend &= ~(1u << u);
          prog = true;
        }
      __syncwarp();
      if (!rdone && cnt[lane] == lrp[lane + 1] - lrp[lane]) {
        // every product of the row is in shared memory: sum in entry order
        T acc = 0;
        for (int q = lrp[lane]; q < lrp[lane + 1]; ++q) acc += prod[q];
        if (kind == 1) {
          st_strong(part + h1.y, acc);
          rdone = true;
        } else {
          bool ready = true;
          if (kind == 2) {  // the partial sums of the row's earlier pieces
            T ps = 0;
            for (int q = h1.y; q < h1.z; ++q) {
              const T pv = ld_strong(part + q);
              ready &= !is_sent(pv);
              ps += pv;
            }
            acc = ps + acc;
          }
          if (ready) {
            const int r = r0 + t0 + lane;
            const T xv = bwr - acc;
            xloc[lane] = xv;
            st_strong(xs + r, xv);
            SF_TRACE(st, r, 1);
            rdone = true;
          }
        }
        prog |= rdone;
      }
      if (__all_sync(0xffffffffu, rdone)) break;
      if (__any_sync(0xffffffffu, prog)) {
        ns = 0;
      } else {
        if (__any_sync(0xffffffffu, wd_giveup(spins, st))) break;
        ns = backoff(ns, st.backoff_ns);
      }
      __syncwarp();
    }
    __syncwarp();  // shared state is rewritten by the next item
  }
}

// The square that follows a triangle in execution order, fused into the
// triangle's kernel as trailing work items (exec.cu fuse_square_items).
struct SqDesc {
  const int* rows;  // DCSR stored rows (dcsr), else rows are row0 + t
  const int* rp;
  const int* ci;
  const void* val;
  int row0, dcsr;
};

// Sync-free, mixed granularity (B200 selector, nrhs == 1; exec.cu
// build_sf_mixed).  Work items in row order, one per ticket (deadlock-free
// like K3):
//   kind 0  a GROUP of <= 32 consecutive rows with <= kSfLong off-diagonal
//           entries each, one lane per row (the thread-per-component form of
//           L247).  A lane consumes its dependencies in batches of U loads;
//           when it meets an unsolved x_j it keeps that ONE address and the
//           warp enters a lean spin (one strong load per blocked lane, a
//           ballot, a branch -- no other issue slots taken from the SM's
//           critical warps) until some lane's value lands.
//   kind 3  a LONG row of <= kSfNB entries, solved by the whole warp (a warp
//           per component, L247): all its loads in flight at once.
//   kind 1/2 the pieces of a row longer than kSfNB: partial sums to `part`
//           slots (sentinel until written), the last piece adds them in piece
//           order (deterministic) and publishes x.
//   kind 4  (fused square, after every triangle item) a block of <= 32
//           stored rows of the NEXT square segment with <= kSfNB entries:
//           b'_rows -= A x, its x_j polled like a triangle's (they are this
//           triangle's rows or earlier ones), products staged in shared
//           memory, lane-per-row sums in entry order (as k::sq_adapt_1);
//   kind 5  a kSfNB-entry chunk of a longer square row (atomic update).
// The fused square's items are claimed only after the triangle's last item,
// i.e. while the triangle's tail leaves most of the GPU idle (the square no
// longer waits for a kernel boundary, and never blocks a triangle row).
#ifndef SPTRSV_SFM_MINB
#define SPTRSV_SFM_MINB 2  // resident CTAs per SM requested from ptxas (3: spills in fp64, measured slower)
#endif
template <typename T, int U>
__global__ void __launch_bounds__(256, SPTRSV_SFM_MINB) tri_sf_mixed(int r0, int nitem, const SfItem* __restrict__ items,
                                                    const int* __restrict__ rp, const int* __restrict__ ci,
                                                    const T* __restrict__ val, T* __restrict__ bw,
                                                    T* __restrict__ xs, T* __restrict__ part, SolveState st,
                                                    int slot, SqDesc sq) {
  constexpr int UW = kSfNB / 32;
  __shared__ T prod_s[8][kSfNB];
  const int lane = threadIdx.x & 31;
  uint32_t* ticket = st.tickets + slot;
  uint32_t spins = 0;
  for (;;) {
    int w = 0;
    if (lane == 0) w = (int)atomicAdd(ticket, 1u);
    w = __shfl_sync(0xffffffffu, w, 0);
    if (w >= nitem) break;
    const int4 h0 = __ldg((const int4*)(items + w));
    const int4 h1 = __ldg((const int4*)(items + w) + 1);
    if (h1.x == 0) {  // ---------------------------------------- row group
      const int k = h0.x + lane;
      bool done = k >= h0.y;
      const int r = r0 + k;
      int p = 0, e = 0;
      T s = 0;
      if (!done) {
        SF_TRACE(st, r, 0);
        p = rp[k];
        e = rp[k + 1];
        s = bw[r];
      }
      int jb = 0;
      T vb = 0, xb = 0;
      bool blocked = false;
      for (;;) {
        if (!done) {
          if (blocked && !is_sent(xb)) {
            s -= vb * xb;
            ++p;
            blocked = false;
          }
          while (!blocked && p < e) {
            const int cnt = min(U, e - p);
            int j[U];
            T v[U], x[U];
#pragma unroll
            for (int u = 0; u < U; ++u)
              if (u < cnt) {
                j[u] = ldg_nc(ci + p + u);
                v[u] = ldg_nc(val + p + u);
              }
#pragma unroll
            for (int u = 0; u < U; ++u)
              if (u < cnt) x[u] = ld_strong(xs + j[u]);
            int took = 0;
#pragma unroll
            for (int u = 0; u < U; ++u)
              if (u < cnt && took == u) {
                if (!is_sent(x[u])) {
                  s -= v[u] * x[u];
                  ++took;
                } else {
                  jb = j[u];
                  vb = v[u];
                  xb = x[u];
                  blocked = true;
                }
              }
            p += took;
          }
          if (!blocked) {
            st_strong(xs + r, s);
            SF_TRACE(st, r, 1);
            done = true;
          }
        }
        if (__all_sync(0xffffffffu, done)) break;
        // lean spin until some blocked lane's value has landed.  kSfPolls
        // polls of the address are in flight at once, issued kSfGap cycles
        // apart and checked in order: the first that sees the value ends the
        // wait, so the detection delay is ~ the poll spacing, not a whole L2
        // round trip (the level's LAST row -- the slowest detection of ~10^3
        // -- sets the level time)
        bool give = false;
        while (!__any_sync(0xffffffffu, !done && !is_sent(xb))) {
          if (__any_sync(0xffffffffu, wd_giveup(spins, st))) {
            give = true;
            break;
          }
          if constexpr (kSfPolls == 1) {
            if (!done) xb = ld_strong(xs + jb);
          } else {
            T xq[kSfPolls];
#pragma unroll
            for (int q = 0; q < kSfPolls; ++q) {
              if (!done) xq[q] = ld_strong(xs + jb);
              if (q + 1 < kSfPolls) {
                const long long t0 = clock64();
                while (clock64() - t0 < kSfGap) {
                }
              }
            }
#pragma unroll
            for (int q = 0; q < kSfPolls; ++q) {
              if (!done && is_sent(xb) && !is_sent(xq[q])) xb = xq[q];
              if (__any_sync(0xffffffffu, !done && !is_sent(xb))) break;
            }
          }
        }
        if (give) break;
      }
      continue;
    }
    if (h1.x >= 4) {  // ------------------------------ fused square block / chunk
      const int a = h0.z, ne = h0.w - h0.z;
      const T* sval = (const T*)sq.val;
      int j[UW];
      T v[UW], x[UW];
      uint32_t pend = 0;
#pragma unroll
      for (int u = 0; u < UW; ++u) {
        const int e = lane + 32 * u;
        if (e < ne) {
          j[u] = ldg_nc(sq.ci + a + e);
          v[u] = ldg_nc(sval + a + e);
        }
      }
#pragma unroll
      for (int u = 0; u < UW; ++u)
        if (lane + 32 * u < ne) x[u] = ld_strong(xs + j[u]);
#pragma unroll
      for (int u = 0; u < UW; ++u)
        if (lane + 32 * u < ne) {
          if (is_sent(x[u])) pend |= 1u << u;
        } else {
          x[u] = T(0);
          v[u] = T(0);
        }
      bool give = false;
      while (__any_sync(0xffffffffu, pend != 0)) {
        if (__any_sync(0xffffffffu, wd_giveup(spins, st))) {
          give = true;
          break;
        }
#pragma unroll
        for (int u = 0; u < UW; ++u)
          if (pend & (1u << u)) {
            x[u] = ld_strong(xs + j[u]);
            if (!is_sent(x[u])) pend &= ~(1u << u);
          }
      }
      if (give) break;
      if (h1.x == 5) {  // chunk of one long stored row
        T acc = 0;
#pragma unroll
        for (int u = 0; u < UW; ++u) acc += v[u] * x[u];
        acc = warp_sum(acc);
        if (lane == 0) atomicAdd(bw + (sq.dcsr ? sq.rows[h0.x] : sq.row0 + h0.x), -acc);
      } else {
        T* pr = prod_s[threadIdx.x >> 5];
#pragma unroll
        for (int u = 0; u < UW; ++u)
          if (lane + 32 * u < ne) pr[lane + 32 * u] = v[u] * x[u];
        __syncwarp();
        const int t = h0.x + lane;
        if (t < h0.y) {
          const int q0 = sq.rp[t] - a, q1 = sq.rp[t + 1] - a;
          if (q1 > q0) {
            T sum = 0;
            for (int q = q0; q < q1; ++q) sum += pr[q];
            bw[sq.dcsr ? sq.rows[t] : sq.row0 + t] -= sum;
          }
        }
        __syncwarp();  // pr is rewritten by the warp's next item
      }
      continue;
    }
    // ------------------------------------------- a long row / a piece of one
    const int kind = h1.x, p0 = h0.z, ne = h0.w - h0.z;
    const int r = r0 + h0.x;
    if (lane == 0) SF_TRACE(st, r, 0);
    const T bwr = (kind != 1 && lane == 0) ? bw[r] : T(0);
    int j[UW];
    T v[UW], x[UW];
    uint32_t pend = 0;
#pragma unroll
    for (int u = 0; u < UW; ++u) {
      const int e = lane + 32 * u;
      if (e < ne) {
        j[u] = ldg_nc(ci + p0 + e);
        v[u] = ldg_nc(val + p0 + e);
      }
    }
#pragma unroll
    for (int u = 0; u < UW; ++u)
      if (lane + 32 * u < ne) {
        x[u] = ld_strong(xs + j[u]);
        if (is_sent(x[u])) pend |= 1u << u;
      } else {
        x[u] = T(0);
        v[u] = T(0);
      }
    bool give = false;
    while (__any_sync(0xffffffffu, pend != 0)) {
      if (__any_sync(0xffffffffu, wd_giveup(spins, st))) {
        give = true;
        break;
      }
#pragma unroll
      for (int u = 0; u < UW; ++u)
        if (pend & (1u << u)) {
          x[u] = ld_strong(xs + j[u]);
          if (!is_sent(x[u])) pend &= ~(1u << u);
        }
    }
    if (give) break;
    T acc = 0;
#pragma unroll
    for (int u = 0; u < UW; ++u) acc += v[u] * x[u];
    acc = warp_sum(acc);
    if (kind == 2) {  // add the earlier pieces' partial sums, 32 at a time, in piece order
      T ps = T(0);   // (a row of > 32 * kSfNB entries has > 32 pieces: the hub columns of
      for (int q0 = h1.y; q0 < h1.z; q0 += 32) {  // C3 become rows of 258K entries in C3^T)
        T pv = T(0);
        if (q0 + lane < h1.z) {
          pv = ld_strong(part + q0 + lane);
          while (is_sent(pv)) {
            if (wd_giveup(spins, st)) break;
            pv = ld_strong(part + q0 + lane);
          }
        }
        ps += warp_sum(pv);
      }
      acc += ps;
    }
    if (lane == 0) {
      if (kind == 1) {
        st_strong(part + h1.y, acc);
      } else {
        st_strong(xs + r, bwr - acc);
        SF_TRACE(st, r, 1);
      }
    }
  }
}

// Sync-free, one WARP per item with a static round-robin schedule (B200
// selector, nrhs == 1; exec.cu build_sf_wrow).  Items are single rows of
// <= 32*UW off-diagonal entries, or kSfW-entry pieces of a longer row
// (kind 1: partial sum to a `part` slot; kind 2: the row's last piece adds
// the earlier pieces' sums in piece order).  Warp w takes items w, w + W,
// w + 2W, ... in order; the launch is cooperative (all W warps resident),
// so the lowest unfinished item always has its owner at it and every
// dependency finished: no deadlock, and no ticket atomics (one same-address
// atomic per row serialised the round-1 warp kernel).  A warp holds ONE
// item: its lanes' loads are all in flight, the warp spins only on its own
// pending dependencies, and nothing else in the warp delays the detection
// (with a row per lane, one lane's next batch stalls the other lanes' polls).
template <typename T, int UW>
__global__ void __launch_bounds__(256) tri_sf_wrow(int r0, int nitem, const SfItem* __restrict__ items,
                                                   const int* __restrict__ ci, const T* __restrict__ val,
                                                   const T* __restrict__ bw, T* __restrict__ xs,
                                                   T* __restrict__ part, SolveState st) {
  const int lane = threadIdx.x & 31;
  const int nw = (gridDim.x * blockDim.x) >> 5;
  uint32_t spins = 0;
  for (int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitem; w += nw) {
    const int4 h0 = __ldg((const int4*)(items + w));
    const int4 h1 = __ldg((const int4*)(items + w) + 1);
    const int kind = h1.x, p0 = h0.z, ne = h0.w - h0.z;
    const int r = r0 + h0.x;
    if (lane == 0) SF_TRACE(st, r, 0);
    const T bwr = (kind != 1 && lane == 0) ? bw[r] : T(0);
    int j[UW];
    T v[UW], x[UW];
#pragma unroll
    for (int u = 0; u < UW; ++u) {
      const int e = lane + 32 * u;
      if (e < ne) {
        j[u] = ldg_nc(ci + p0 + e);
        v[u] = ldg_nc(val + p0 + e);
      }
    }
    uint32_t pend = 0;
#pragma unroll
    for (int u = 0; u < UW; ++u)
      if (lane + 32 * u < ne) x[u] = ld_strong(xs + j[u]);
#pragma unroll
    for (int u = 0; u < UW; ++u)
      if (lane + 32 * u < ne) {
        if (is_sent(x[u])) pend |= 1u << u;
      } else {
        x[u] = T(0);
        v[u] = T(0);
      }
    bool give = false;
    while (__any_sync(0xffffffffu, pend != 0)) {
#pragma unroll
      for (int u = 0; u < UW; ++u)
        if (pend & (1u << u)) x[u] = ld_strong(xs + j[u]);
#pragma unroll
      for (int u = 0; u < UW; ++u)
        if ((pend & (1u << u)) && !is_sent(x[u])) pend &= ~(1u << u);
      if (__any_sync(0xffffffffu, wd_giveup(spins, st))) {
        give = true;
        break;
      }
    }
    if (give) break;
    T acc = 0;
#pragma unroll
    for (int u = 0; u < UW; ++u) acc += v[u] * x[u];
    acc = warp_sum(acc);
    if (kind == 2) {  // the earlier pieces' partial sums, 32 at a time, in piece order
      T ps = T(0);
      for (int q0 = h1.y; q0 < h1.z; q0 += 32) {
        T pv = T(0);
        if (q0 + lane < h1.z) {
          pv = ld_strong(part + q0 + lane);
          while (is_sent(pv)) {
            if (wd_giveup(spins, st)) break;
            pv = ld_strong(part + q0 + lane);
          }
        }
        ps += warp_sum(pv);
      }
      acc += ps;
    }
    if (lane == 0) {
      if (kind == 1) {
        st_strong(part + h1.y, acc);
      } else {
        st_strong(xs + r, bwr - acc);
        SF_TRACE(st, r, 1);
      }
    }
  }
}

// Supernodal sync-free (B200 selector, nrhs == 1): a warp per fundamental
// supernode piece J = rows [s, s+w), w <= 32, claimed in row order from the
// segment's ticket (deadlock-free like K3).  Lane t owns row s+t:
//   1. y_t = b'_t - sum_q V_J[t][q] x_{E_J[q]}: the piece's rows share one
//      list E_J of external columns, so 32 columns per round are polled by
//      32 lanes (value-as-flag), broadcast by shuffles, and met by a
//      coalesced column of V_J (loaded before the poll);
//   2. x = T_J^{-1} y for the dense unit-lower diagonal block T_J (after the
//      D^-1 scaling, R27): w-1 steps of shfl x_c -> DFMA, lane t's row of
//      T_J in registers;
//   3. x_t stored with a strong store, which publishes it (value-as-flag).
// The critical path is one dependency hop per PIECE instead of one per row
// (a 64-wide supernode is 64 levels of the row DAG).
struct SnDesc {
  int s, w, ne, coff;          // first global row, width, |E_J|, offset of E_J in cols
  long long voff, boff;        // offsets (elements) of V_J and of the packed T_J
};

#ifndef SPTRSV_SN_MINB
#define SPTRSV_SN_MINB 2  // min resident CTAs per SM requested from ptxas (C4: 2 measured best of 1-3)
#endif
// Work items (exec.cu build_supernodes): a piece whose external column list
// is longer than kSnChunk is cut into kSnChunk-column chunks -- partial
// products V_J[:, chunk] x[chunk] go to 32-wide slots of `part` (sentinel
// until written), and the piece's last chunk adds them in chunk order
// (deterministic) before the diagonal block.  The pieces near the root of
// the elimination tree hold the longest lists (all their children's and
// grandchildren's columns) and sit at the END of the dependency chain: split,
// their products run on many warps at once instead of one warp's serial rounds.
#ifndef SPTRSV_SN_CHUNK
#define SPTRSV_SN_CHUNK 256
#endif
constexpr int kSnChunk = SPTRSV_SN_CHUNK;
struct SnItem {
  int J, q0, q1, kind;  // piece, external columns [q0, q1); kind 0 whole piece, 1 partial chunk, 2 last chunk
  int s0, s1, pad0, pad1;  // kind 1: slot s0; kind 2: slots [s0, s1)
};
template <typename T>
__global__ void __launch_bounds__(256, SPTRSV_SN_MINB) tri_supernode(int nitems, const SnItem* __restrict__ items,
                                                     const SnDesc* __restrict__ desc,
                                                     const int* __restrict__ cols, const T* __restrict__ V,
                                                     const T* __restrict__ Tb, const T* __restrict__ bw,
                                                     T* __restrict__ xs, T* __restrict__ part, SolveState st,
                                                     int slot) {
  const int lane = threadIdx.x & 31;
  uint32_t* ticket = st.tickets + slot;
  while (true) {
    int w = 0;
    if (lane == 0) w = (int)atomicAdd(ticket, 1u);
    w = __shfl_sync(0xffffffffu, w, 0);
    if (w >= nitems) break;
    const int4 i0 = __ldg((const int4*)(items + w));
    const int4 i1 = __ldg((const int4*)(items + w) + 1);
    const int kind = i0.w;
    const SnDesc d = desc[i0.x];
    const bool act = lane < d.w;
    // kind 0 / 2: y = b' - V x; kind 1: y = V x over the chunk (a partial)
    T y = (act && kind != 1) ? bw[d.s + lane] : T(0);
    if (kind == 1) y = T(0);
    for (int q0 = i0.y; q0 < i0.z; q0 += 32) {
      const int nq = min(32, i0.z - q0);
      const bool inq = lane < nq;
      const int j = inq ? ldg_nc(cols + d.coff + q0 + lane) : 0;
      T vr[32];
      const T* Vq = V + d.voff + (long long)q0 * d.w + lane;
#pragma unroll
      for (int c = 0; c < 32; ++c) vr[c] = (c < nq && act) ? ldg_nc(Vq + (long long)c * d.w) : T(0);
      T xj = inq ? ld_strong(xs + j) : T(0);
      uint32_t spins = 0;
      unsigned ns = 0;
      while (__any_sync(0xffffffffu, inq && is_sent(xj))) {
        if (__any_sync(0xffffffffu, wd_giveup(spins, st))) break;
        ns = backoff(ns, st.backoff_ns);
        if (inq && is_sent(xj)) xj = ld_strong(xs + j);
      }
#pragma unroll
      for (int c = 0; c < 32; ++c) {
        if (c < nq) {  // warp-uniform
          const T xc = __shfl_sync(0xffffffffu, xj, c);
          if (kind == 1)
            y += vr[c] * xc;
          else
            y -= vr[c] * xc;
        }
      }
    }
    if (kind == 1) {  // publish the chunk's partial products (32-wide slot)
      if (act) st_strong(part + (size_t)i1.x * 32 + lane, y);
      continue;
    }
    if (kind == 2) {  // the earlier chunks' partials, in chunk order
      T ps = T(0);
      for (int q = i1.x; q < i1.y; ++q) {
        T pv = act ? ld_strong(part + (size_t)q * 32 + lane) : T(0);
        uint32_t spins = 0;
        while (__any_sync(0xffffffffu, act && is_sent(pv))) {
          if (__any_sync(0xffffffffu, wd_giveup(spins, st))) break;
          if (act && is_sent(pv)) pv = ld_strong(part + (size_t)q * 32 + lane);
        }
        ps += pv;
      }
      y -= ps;
    }
    // dense unit-lower diagonal block: column c of T_J holds rows c+1 .. w-1
    // at Tb[boff + c(w-1) - c(c-1)/2 + (t - c - 1)]
    T tl[31];
#pragma unroll
    for (int c = 0; c < 31; ++c) {
      const long long off = d.boff + (long long)c * (d.w - 1) - (long long)c * (c - 1) / 2 + (lane - c - 1);
      tl[c] = (act && lane > c && c < d.w - 1) ? ldg_nc(Tb + off) : T(0);
    }
#pragma unroll
    for (int c = 0; c < 31; ++c) {
      if (c < d.w - 1) {  // warp-uniform
        const T xc = __shfl_sync(0xffffffffu, y, c);
        y -= tl[c] * xc;  // lanes <= c hold tl[c] = 0
      }
    }
    if (act) st_strong(xs + d.s + lane, y);
  }
}

// Supernodal SpTRSM (B200 selector, nrhs >= 16): a CTA per
// supernode piece J = rows [s, s+w), w <= 32, claimed in row order from the
// segment's ticket, and the RHS in chunks of 64 columns.  Per chunk:
//   1. Y = B'_J - V_J X[E_J, :] as a register-tiled dense product: the 32
//      external columns of a round are polled (per-row epoch flags, one thread
//      each), their X rows (32 x 64) and the matching V_J panel (32 x w) are
//      staged in shared memory, and warp wi accumulates rows 4wi..4wi+3 x 64
//      columns (lane and lane+32): 8 DFMA per 4 shared loads, V_J read once
//      per chunk instead of once per RHS column;
//   2. X_J = T_J^{-1} Y for the dense unit-lower diagonal block: warp wi owns
//      8 columns, lane t row t, 31 shfl/DFMA steps with T_J's row in registers;
//   3. X_J stored coalesced; after the last chunk the piece's row flags are
//      published (fence, barrier, flag = epoch).
// In fp64 on B200 the DMMA tensor-core rate is not above the DFMA rate, so
// the dense tiles run on the FMA pipes (f-3).
constexpr int kSnmCols = 64;
constexpr int kSnmXld = kSnmCols + 4;
#ifndef SPTRSV_SNM_DMMA
#define SPTRSV_SNM_DMMA 1
#endif

// fp64 tensor-core MMA (DMMA, mma.sync m8n8k4 .f64 -- tcgen05 has no f64
// kind, so this is sm_100a's f64 tensor-core path): D = A(8x4, row) x
// B(4x8, col) + C.  Fragments (g = lane >> 2, q = lane & 3): a = A[g][q],
// b = B[q][g], c/d = {C[g][2q], C[g][2q+1]}.
__device__ __forceinline__ void dmma_8x8x4(double& d0, double& d1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};"
               : "+d"(d0), "+d"(d1)
               : "d"(a), "d"(b));
}
template <typename T>
__global__ void __launch_bounds__(256, 4) tri_supernode_multi(int npieces, const SnDesc* __restrict__ desc,
                                                           const int* __restrict__ cols, const T* __restrict__ V,
                                                           const T* __restrict__ Tb, const T* __restrict__ bw,
                                                           T* __restrict__ xs, SolveState st, int slot, int nrhs,
                                                           int c_lo, int c_hi) {
  __shared__ __align__(16) T Vs[32][32];
  __shared__ __align__(16) T Xs[32][kSnmXld];  // row pad: the DMMA B fragments read 4 rows x 8 columns
  __shared__ __align__(16) T Ys[32][kSnmCols + 1];
  __shared__ int Js[2][32];
  __shared__ int Jsh;
  constexpr bool kSnmDmma = sizeof(T) == 8 && SPTRSV_SNM_DMMA;  // fp64 product on the tensor cores
  const int tid = threadIdx.x, lane = tid & 31, wi = tid >> 5;
  uint32_t* ticket = st.tickets + slot;
  const uint32_t epoch = solve_epoch(st);
  while (true) {
    if (tid == 0) Jsh = (int)atomicAdd(ticket, 1u);
    __syncthreads();
    const int J = Jsh;
    __syncthreads();  // Jsh is rewritten by the next claim
    if (J >= npieces) break;
    const SnDesc d = desc[J];
    for (int c0 = c_lo; c0 < c_hi; c0 += kSnmCols) {
      // fp64: warp wi owns the 8 x 8 DMMA tiles (row block wi & 3, column
      // blocks 4 (wi >> 2) .. +3); acc[i][u] = C[t = 8 rb + g][c = 8 cb_i + 2 q + u].
      // fp32: warp wi owns rows 4 wi .. 4 wi + 3, lane columns lane, lane + 32.
      T acc[4][2];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          const int t = kSnmDmma ? 8 * (wi & 3) + (lane >> 2) : wi * 4 + i;
          const int c = c0 + (kSnmDmma ? 8 * (4 * (wi >> 2) + i) + 2 * (lane & 3) + u : lane + 32 * u);
          acc[i][u] = (t < d.w && c < nrhs) ? bw[(int64_t)(d.s + t) * nrhs + c] : T(0);
        }
      // round prologue for external columns [q0, q0+32): one thread per
      // column loads its index into Js[buf] and (first chunk only) polls its
      // epoch flag; every thread loads its part of the V_J panel to registers
      T vr[4];
      auto prep = [&](int q0, int buf) {
        const int nq = min(32, d.ne - q0);
        if (tid < nq) {
          const int j = ldg_nc(cols + d.coff + q0 + tid);
          Js[buf][tid] = j;
          if (c0 == c_lo) {  // later column chunks find the rows already published
            uint32_t spins = 0;
            unsigned ns = 0;
            while (ld_flag(st.flags + j) != epoch) {
              if (wd_giveup(spins, st)) break;
              ns = backoff(ns, st.backoff_ns);
            }
            __threadfence();
          }
        }
        const T* Vq = V + d.voff + (long long)q0 * d.w;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const int q = (tid >> 5) + 8 * k, t = tid & 31;
          vr[k] = (q < nq && t < d.w) ? ldg_nc(Vq + (long long)q * d.w + t) : T(0);
        }
      };
      prep(0, 0);
      __syncthreads();  // Js[0] and the readiness of its rows
      // two barriers per round: the next round's prologue runs between the
      // product and the barrier that ends the round (Js is double-buffered;
      // Vs / Xs are rewritten only after that barrier)
      for (int q0 = 0, buf = 0; q0 < d.ne; q0 += 32, buf ^= 1) {
        const int nq = min(32, d.ne - q0);
        // all staging loads of a round are issued before any shared store
        // (ld_strong is an asm volatile with a memory clobber: interleaved
        // with the stores it would serialise on the load latency)
        T xr[32 * kSnmCols / 256];
#pragma unroll
        for (int k = 0; k < 32 * kSnmCols / 256; ++k) {
          const int idx = tid + 256 * k, q = idx / kSnmCols, c = idx % kSnmCols;
          xr[k] = (q < nq && c0 + c < nrhs) ? ld_strong(xs + (int64_t)Js[buf][q] * nrhs + c0 + c) : T(0);
        }
#pragma unroll
        for (int k = 0; k < 4; ++k) Vs[(tid >> 5) + 8 * k][tid & 31] = vr[k];
#pragma unroll
        for (int k = 0; k < 32 * kSnmCols / 256; ++k) {
          const int idx = tid + 256 * k;
          Xs[idx / kSnmCols][idx % kSnmCols] = xr[k];
        }
        __syncthreads();
        if constexpr (kSnmDmma) {
          // C -= V_J^T[rows, q0..q0+32) X[q0..q0+32, cols] on the fp64 tensor
          // cores: 8 k-steps of 4 external columns (rounds are zero-padded)
          const int g = lane >> 2, qq = lane & 3, rb = wi & 3, cb = 4 * (wi >> 2);
#pragma unroll
          for (int k0 = 0; k0 < 32; k0 += 4) {
            if (k0 < nq) {  // CTA-uniform
              const double a = -Vs[k0 + qq][8 * rb + g];
#pragma unroll
              for (int i = 0; i < 4; ++i) dmma_8x8x4(acc[i][0], acc[i][1], a, Xs[k0 + qq][8 * (cb + i) + g]);
            }
          }
        } else {
          for (int q = 0; q < nq; ++q) {
            const T x0 = Xs[q][lane], x1 = Xs[q][lane + 32];
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              const T v = Vs[q][wi * 4 + i];
              acc[i][0] -= v * x0;
              acc[i][1] -= v * x1;
            }
          }
        }
        if (q0 + 32 < d.ne) prep(q0 + 32, buf ^ 1);
        __syncthreads();  // Vs / Xs are restaged next round, Js[buf ^ 1] is ready
      }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          if constexpr (kSnmDmma)
            Ys[8 * (wi & 3) + (lane >> 2)][8 * (4 * (wi >> 2) + i) + 2 * (lane & 3) + u] = acc[i][u];
          else
            Ys[wi * 4 + i][lane + 32 * u] = acc[i][u];
        }
      // T_J column-major in shared memory (aliasing Xs, free after the
      // product): column c holds rows c+1 .. w-1 (packed as in tri_supernode)
      T(*Ts)[32] = reinterpret_cast<T(*)[32]>(&Xs[0][0]);
      for (int idx = tid; idx < 32 * 32; idx += 256) {
        const int c = idx >> 5, t = idx & 31;
        const long long off = d.boff + (long long)c * (d.w - 1) - (long long)c * (c - 1) / 2 + (t - c - 1);
        Ts[c][t] = (t < d.w && t > c && c < d.w - 1) ? ldg_nc(Tb + off) : T(0);
      }
      __syncthreads();
      T y[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) y[i] = Ys[lane][wi * 8 + i];
#pragma unroll 4
      for (int c = 0; c < d.w - 1; ++c) {  // CTA-uniform
        const T tc = Ts[c][lane];          // lanes <= c read 0
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const T xc = __shfl_sync(0xffffffffu, y[i], c);
          y[i] -= tc * xc;
        }
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) Ys[lane][wi * 8 + i] = y[i];
      __syncthreads();
      for (int idx = tid; idx < 32 * kSnmCols; idx += 256) {
        const int t = idx / kSnmCols, c = idx % kSnmCols;
        if (t < d.w && c0 + c < nrhs) xs[(int64_t)(d.s + t) * nrhs + c0 + c] = Ys[t][c];
      }
      __syncthreads();  // Ys is rewritten by the next chunk
    }
    __threadfence();  // the piece's x stores are visible at gpu scope ...
    __syncthreads();
    if (tid < d.w) st_flag(st.flags + d.s + tid, epoch);  // ... before its row flags
  }
}

// Multi-RHS sync-free (SpTRSM): a group of G lanes per component, lanes over
// the RHS columns.  Readiness is a per-row flag holding the solve's epoch
// (no per-solve reset, no n x nrhs sentinel fill): the G lanes store the row,
// each fences (membar.gl), the group syncs, lane 0 publishes the flag; a
// reader polls the flag and then reads the row with strong (L2) loads.
template <typename T, int G, int RPT>
__global__ void __launch_bounds__(256) tri_syncfree_multi(int r0, int m, const int* __restrict__ rp,
                                                          const int* __restrict__ ci, const T* __restrict__ val,
                                                          const T* __restrict__ bw, T* __restrict__ xs,
                                                          SolveState st, int slot, int nrhs) {
  const int lane = threadIdx.x % G;
  const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << ((threadIdx.x & 31) / G * G));
  uint32_t* ticket = st.tickets + slot;
  const uint32_t epoch = solve_epoch(st);
  while (true) {
    int k = 0;
    if (lane == 0) k = (int)atomicAdd(ticket, 1u);
    k = __shfl_sync(gmask, k, 0, G);
    if (k >= m) break;
    const int r = r0 + k;
    const int a = rp[k], e = rp[k + 1];
    for (int c0 = 0; c0 < nrhs; c0 += G * RPT) {
      // a whole pass of columns in range: with one predicate per column the
      // 7 predicate registers run out and ptxas interleaves FMAs with the
      // gathers (9 of 16 in flight; C5 seg0 3.5 -> 8.3 ms in round 2)
      const bool full = c0 + G * RPT <= nrhs;
      T acc[RPT];
#pragma unroll
      for (int t = 0; t < RPT; ++t)
        acc[t] = (c0 + lane + G * t < nrhs) ? bw[(int64_t)r * nrhs + c0 + lane + G * t] : T(0);
      for (int p = a; p < e; ++p) {
        const int j = ldg_nc(ci + p);
        const T v = ldg_nc(val + p);
        if (c0 == 0) {  // later column chunks of this row find j already published
          uint32_t spins = 0;
          unsigned ns = 0;
          while (ld_flag(st.flags + j) != epoch) {
            if (wd_giveup(spins, st)) break;
            ns = backoff(ns, st.backoff_ns);
          }
        }
        const T* xr = xs + (int64_t)j * nrhs + c0 + lane;
        T x[RPT];
        if (full) {  // no per-column predicates: all RPT gathers issue before the first FMA
#pragma unroll
          for (int t = 0; t < RPT; ++t) x[t] = ld_strong(xr + G * t);
#pragma unroll
          for (int t = 0; t < RPT; ++t) acc[t] -= v * x[t];
        } else {
#pragma unroll
          for (int t = 0; t < RPT; ++t)
            if (c0 + lane + G * t < nrhs) x[t] = ld_strong(xr + G * t);
#pragma unroll
          for (int t = 0; t < RPT; ++t)
            if (c0 + lane + G * t < nrhs) acc[t] -= v * x[t];
        }
      }
      T* xo = xs + (int64_t)r * nrhs + c0 + lane;
#pragma unroll
      for (int t = 0; t < RPT; ++t)
        if (c0 + lane + G * t < nrhs) xo[G * t] = acc[t];
    }
    __threadfence();  // this lane's x stores are visible at gpu scope ...
    __syncwarp(gmask);
    if (lane == 0) st_flag(st.flags + r, epoch);  // ... before the row's flag
  }
}

// ------------------------------------- K4 (staged): TMA-fed single-CTA chain
// The level walk of tri_chain_1, but the triangle's CSR rows stream into
// shared memory ahead of the walk with cp.async.bulk (TMA) copies that
// complete on mbarriers, and solved x values stay in a shared-memory ring
// window, so the per-level critical path is bar.sync -> ld.shared x_j -> FMA
// chain -> st.shared x_i, with no global memory on it.
//
// Stage s (a record computed by the analysis) covers local rows [sa, sb) --
// whole levels where possible -- with their entries [e0, e1) and level
// pointers lp[l0 .. l0+nl-1].  recs[2s] is stage s's record and recs[2s+1]
// the record of stage s+NST; both travel in stage s's buffer, so neither the
// consumers nor the producer (thread 0) touch global memory for control.
struct StageRec {
  int sa, sb, e0, e1, l0, nl, pad0, pad1;
};

__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(smem_addr(bar)), "r"(parity)
        : "memory");
  }
}
__device__ __forceinline__ void tma_bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_addr(dst)),
               "l"(src), "r"(bytes), "r"(smem_addr(bar))
               : "memory");
}

struct ChainGeom {
  int NST, RMAX, EMAX, XW, LMAX;
  uint32_t cap_rp, cap_ci, cap_val, cap_v, cap_lp, stage_bytes;
};

__host__ __device__ inline uint32_t al16(uint32_t v) { return (v + 15u) & ~15u; }

template <typename T>
__host__ __device__ inline ChainGeom chain_geom(int NST, int RMAX, int EMAX, int XW, int LMAX) {
  ChainGeom g;
  g.NST = NST;
  g.RMAX = RMAX;
  g.EMAX = EMAX;
  g.XW = XW;
  g.LMAX = LMAX;
  g.cap_rp = al16((RMAX + 8) * 4);
  g.cap_ci = al16((EMAX + 8) * 4);
  g.cap_val = al16((EMAX + 4) * (uint32_t)sizeof(T));
  g.cap_v = al16((RMAX + 4) * (uint32_t)sizeof(T));
  g.cap_lp = al16((LMAX + 8) * 4);
  g.stage_bytes = 64 + g.cap_rp + g.cap_ci + g.cap_val + g.cap_v + g.cap_lp;
  return g;
}
template <typename T>
__host__ __device__ inline uint32_t chain_smem_bytes(const ChainGeom& g) {
  return g.NST * g.stage_bytes + g.XW * (uint32_t)sizeof(T) + g.NST * 16;  // + full/empty mbarriers
}

// 16-byte aligned window around element range [first, first+count)
struct Win {
  const char* src;
  uint32_t bytes;
};
template <typename E>
__device__ __forceinline__ Win win(const E* base, int64_t first, int64_t count) {
  uintptr_t a = (uintptr_t)(base + first);
  uintptr_t lo = a & ~(uintptr_t)15;
  uintptr_t hi = ((uintptr_t)(base + first + count) + 15) & ~(uintptr_t)15;
  return Win{(const char*)lo, (uint32_t)(hi - lo)};
}
template <typename E>
__device__ __forceinline__ int shift_of(const E* base, int64_t first) {
  return (int)(((uintptr_t)(base + first) & 15) / sizeof(E));
}

template <typename T>
__global__ void __launch_bounds__(1024, 1)
    tri_chain_tma(int r0, int nstage, const StageRec* __restrict__ recs, const int* __restrict__ lp,
                  const int* __restrict__ rp, const int* __restrict__ ci, const T* __restrict__ val,
                  const T* __restrict__ bw, T* __restrict__ xs, ChainGeom g, long long* __restrict__ trace) {
  // Warp-specialised: the last warp is the TMA producer, the other warps
  // (NC threads) walk the levels and synchronise on named barrier 1, so the
  // copy issue never sits on the dependency chain.
  extern __shared__ __align__(128) unsigned char smem[];
  const int tid = threadIdx.x;
  const int NC = blockDim.x - 32;
  const int xmask = g.XW - 1;  // XW is a power of two
  T* xw = (T*)(smem + g.NST * g.stage_bytes);
  uint64_t* full = (uint64_t*)(smem + g.NST * g.stage_bytes + g.XW * sizeof(T));
  uint64_t* empty = full + g.NST;
  if (tid == 0) {
    for (int b = 0; b < g.NST; ++b) {
      mbar_init(&full[b], 1);
      mbar_init(&empty[b], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  struct Bufs {
    StageRec* rec;
    int* rp;
    int* ci;
    T* val;
    T* b;
    int* lp;
  };
  auto bufs = [&](int b) {
    unsigned char* base = smem + (size_t)b * g.stage_bytes;
    Bufs B;
    B.rec = (StageRec*)base;
    B.rp = (int*)(base + 64);
    B.ci = (int*)(base + 64 + g.cap_rp);
    B.val = (T*)(base + 64 + g.cap_rp + g.cap_ci);
    B.b = (T*)(base + 64 + g.cap_rp + g.cap_ci + g.cap_val);
    B.lp = (int*)(base + 64 + g.cap_rp + g.cap_ci + g.cap_val + g.cap_v);
    return B;
  };

  if (tid >= NC) {  // ---------------- producer warp
    if (tid == NC) {
      int b = 0;
      uint32_t ph = 0;
      for (int s = 0; s < nstage; ++s) {
        Bufs B = bufs(b);
        StageRec R;
        if (s < g.NST) {
          R = recs[2 * s];
        } else {
          mbar_wait(&empty[b], ph ^ 1u);  // consumers released stage s - NST
          R = B.rec[1];                   // stage s's record rode in with stage s - NST
        }
        Win wr = win(rp, R.sa, R.sb - R.sa + 1);
        Win wc = win(ci, R.e0, R.e1 - R.e0);
        Win wv = win(val, R.e0, R.e1 - R.e0);
        Win wb = win(bw, (int64_t)r0 + R.sa, R.sb - R.sa);
        Win wl = win(lp, R.l0, R.nl);
        const bool ents = R.e1 > R.e0;
        uint32_t tot = 64 + wr.bytes + wb.bytes + wl.bytes + (ents ? wc.bytes + wv.bytes : 0u);
        mbar_expect_tx(&full[b], tot);
        tma_bulk_g2s(B.rec, recs + 2 * s, 64, &full[b]);
        tma_bulk_g2s(B.rp, wr.src, wr.bytes, &full[b]);
        if (ents) {
          tma_bulk_g2s(B.ci, wc.src, wc.bytes, &full[b]);
          tma_bulk_g2s(B.val, wv.src, wv.bytes, &full[b]);
        }
        tma_bulk_g2s(B.b, wb.src, wb.bytes, &full[b]);
        tma_bulk_g2s(B.lp, wl.src, wl.bytes, &full[b]);
        if (++b == g.NST) {
          b = 0;
          ph ^= 1u;
        }
      }
    }
    return;
  }

  // ---------------- consumer warps
  int b = 0;
  uint32_t ph = 0;
  for (int s = 0; s < nstage; ++s) {
    long long t0 = 0;
    if (trace && tid == 0) t0 = clock64();
    mbar_wait(&full[b], ph);
    if (trace && tid == 0) {
      trace[3 * s] = t0;
      trace[3 * s + 1] = clock64();
    }
    const Bufs B = bufs(b);
    const StageRec R = B.rec[0];
    const int* s_rp = B.rp + shift_of(rp, R.sa);
    const int* s_ci = B.ci + shift_of(ci, R.e0);
    const T* s_val = B.val + shift_of(val, R.e0);
    const T* s_b = B.b + shift_of(bw, (int64_t)r0 + R.sa);
    const int* s_lp = B.lp + shift_of(lp, R.l0);
    for (int li = 0; li + 1 < R.nl; ++li) {
      const int L0 = s_lp[li], L1 = s_lp[li + 1];
      const int la = max(L0, R.sa), lb = min(L1, R.sb);
      const int xlo = L1 - g.XW;  // deps >= xlo are in the window
      for (int r = la + tid; r < lb; r += NC) {
        const int i = r - R.sa;
        const int p0 = s_rp[i] - R.e0, p1 = s_rp[i + 1] - R.e0;
        T acc = s_b[i];
        int p = p0;
        for (; p + 1 < p1; p += 2) {  // two independent dependency loads in flight
          const int j0 = s_ci[p] - r0, j1 = s_ci[p + 1] - r0;
          const T v0 = s_val[p], v1 = s_val[p + 1];
          const T x0 = j0 >= xlo ? xw[j0 & xmask] : xs[r0 + j0];
          const T x1 = j1 >= xlo ? xw[j1 & xmask] : xs[r0 + j1];
          acc -= v0 * x0;
          acc -= v1 * x1;
        }
        if (p < p1) {
          const int j0 = s_ci[p] - r0;
          const T x0 = j0 >= xlo ? xw[j0 & xmask] : xs[r0 + j0];
          acc -= s_val[p] * x0;
        }
        xw[r & xmask] = acc;
        xs[r0 + r] = acc;
      }
      // level barrier (Alg 2 L96) -- also at a stage end that splits a
      // level, so the buffer can be released below
      asm volatile("bar.sync 1, %0;" ::"r"(NC) : "memory");
    }
    if (trace && tid == 0) trace[3 * s + 2] = clock64();
    if (tid == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(&empty[b])) : "memory");
    if (++b == g.NST) {
      b = 0;
      ph ^= 1u;
    }
  }
}

// ------------------------- K4 (staged, ELL): narrow rows, window-resident deps
// When every row of a chain triangle has at most K dependencies and every
// dependency lies inside the x window of its level (both checked by the
// analysis), the triangle is cut into STEPS (a level, or a chunk of a level
// wider than the CTA's row capacity) and every step into groups of 32 rows.
// Step q's group gi is owned by consumer warp gi % NW (gi / NW < RG), lane l
// owns row row_start(q) + 32 gi + l.  Per padded row a stage ships its K
// dependency WINDOW SLOTS (u16, two per word; slot XW is a zero) and K
// values, so one row is: LDS x_j (K, addresses computed before the barrier)
// -> K DFMA -> STS x_i.  Consequences:
//   * no row pointers, level pointers, bounds or modulo on the dependency
//     chain; the per-step overhead is one 16-byte step record (broadcast);
//   * the operands of step q+1 are loaded into registers before step q's
//     barrier (software pipeline across levels);
//   * x never goes to global memory from the consumers: when a stage is
//     done, the producer warp copies its rows from the window to xs with one
//     cp.async.bulk shared->global store (stages never wrap the window).
struct EllRec {
  int sa, sb, nsteps, off16, bytes, npad, pad0, pad1;  // off16: stage block offset in 16-byte units
};

__host__ __device__ inline uint32_t ell_words(int K) { return (uint32_t)(K + 1) / 2; }

template <typename T>
__host__ __device__ inline uint32_t ell_stage_bytes(int K, int RMAX, int PMAX, int SMAX) {
  return 64 + 16u * SMAX + al16(ell_words(K) * PMAX * 4) + al16(K * PMAX * (uint32_t)sizeof(T)) +
         al16((RMAX + 4) * (uint32_t)sizeof(T));
}

__device__ __forceinline__ double lds_x(uint32_t a, double) {
  double v;
  asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ float lds_x(uint32_t a, float) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts_x(uint32_t a, double v) {
  asm volatile("st.shared.f64 [%0], %1;" ::"r"(a), "d"(v) : "memory");
}
__device__ __forceinline__ void sts_x(uint32_t a, float v) {
  asm volatile("st.shared.f32 [%0], %1;" ::"r"(a), "f"(v) : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* dst, uint32_t src_smem, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(src_smem), "r"(bytes)
               : "memory");
}

template <typename T, int K, int RG>
__global__ void __launch_bounds__(1024, 1)
    tri_chain_ell(int r0, int nstage, const EllRec* __restrict__ recs, const char* __restrict__ ell,
                  const T* __restrict__ bw, T* __restrict__ xs, int NST, int RMAX, int PMAX, int SMAX, int XW,
                  long long* __restrict__ trace) {
  extern __shared__ __align__(128) unsigned char smem[];
  constexpr int W = (K + 1) / 2;
  constexpr uint32_t SH = sizeof(T) == 8 ? 3 : 2;
  const int tid = threadIdx.x;
  const int NC = blockDim.x - 32;
  const int NW = NC >> 5, warp = tid >> 5, lane = tid & 31;
  const uint32_t xmask = (uint32_t)XW - 1;
  const uint32_t sbytes = ell_stage_bytes<T>(K, RMAX, PMAX, SMAX);
  const uint32_t o_b = 64 + 16u * SMAX + al16(W * PMAX * 4) + al16(K * PMAX * (uint32_t)sizeof(T));
  unsigned char* xw_p = smem + (size_t)NST * sbytes;  // XW slots + one zero slot
  const uint32_t xw = smem_addr(xw_p);
  uint64_t* full = (uint64_t*)(xw_p + al16((XW + 2) * (uint32_t)sizeof(T)));
  uint64_t* empty = full + NST;
  if (tid == 0) {
    for (int b = 0; b < NST; ++b) {
      mbar_init(&full[b], 1);
      mbar_init(&empty[b], 1);
    }
    ((T*)xw_p)[XW] = T(0);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  if (tid >= NC) {  // ---------------- producer warp: stage loads and x stores
    if (tid == NC) {
      for (int s = 0; s < nstage && s < NST; ++s) {
        unsigned char* B = smem + (size_t)s * sbytes;
        const EllRec R = recs[2 * s];
        Win wb = win(bw, (int64_t)r0 + R.sa, R.sb - R.sa);
        mbar_expect_tx(&full[s], 64 + R.bytes + wb.bytes);
        tma_bulk_g2s(B, recs + 2 * s, 64, &full[s]);
        tma_bulk_g2s(B + 64, ell + (size_t)R.off16 * 16, R.bytes, &full[s]);
        tma_bulk_g2s(B + o_b, wb.src, wb.bytes, &full[s]);
      }
      int b = 0;
      uint32_t ph = 0;
      for (int s = 0; s < nstage; ++s) {
        unsigned char* B = smem + (size_t)b * sbytes;
        mbar_wait(&empty[b], ph);  // stage s solved (its window rows final)
        const EllRec R = ((const EllRec*)B)[0];
        // x rows [sa, sb) of the stage: window slots are contiguous (no wrap)
        int g0 = r0 + R.sa, g1 = r0 + R.sb;
        const T* xwT = (const T*)xw_p;
        if (g0 & 1 && sizeof(T) == 8) {  // 16-byte alignment of the bulk copy
          xs[g0] = xwT[(uint32_t)g0 & xmask];
          ++g0;
        }
        if (sizeof(T) == 4) {
          while ((g0 & 3) && g0 < g1) {
            xs[g0] = xwT[(uint32_t)g0 & xmask];
            ++g0;
          }
        }
        const int per16 = 16 / (int)sizeof(T);
        int g1a = g0 + (g1 - g0) / per16 * per16;
        for (int g = g1a; g < g1; ++g) xs[g] = xwT[(uint32_t)g & xmask];
        if (g1a > g0) {
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          bulk_s2g(xs + g0, xw + (((uint32_t)g0 & xmask) << SH), (uint32_t)(g1a - g0) * sizeof(T));
          asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
        if (s + NST < nstage) {
          // the stores must have read their window slots before the
          // consumers can reach stage s + NST + 1 (which needs the load below)
          asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
          const EllRec Rn = ((const EllRec*)B)[1];  // rode in with stage s
          Win wb = win(bw, (int64_t)r0 + Rn.sa, Rn.sb - Rn.sa);
          mbar_expect_tx(&full[b], 64 + Rn.bytes + wb.bytes);
          tma_bulk_g2s(B, recs + 2 * (s + NST), 64, &full[b]);
          tma_bulk_g2s(B + 64, ell + (size_t)Rn.off16 * 16, Rn.bytes, &full[b]);
          tma_bulk_g2s(B + o_b, wb.src, wb.bytes, &full[b]);
        }
        if (++b == NST) {
          b = 0;
          ph ^= 1u;
        }
      }
      asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    }
    return;
  }

  // ---------------- consumer warps
  int b = 0;
  uint32_t ph = 0;
  for (int s = 0; s < nstage; ++s) {
    long long t0 = 0;
    if (trace && tid == 0) t0 = clock64();
    mbar_wait(&full[b], ph);
    if (trace && tid == 0) {
      trace[3 * s] = t0;
      trace[3 * s + 1] = clock64();
    }
    const unsigned char* B = smem + (size_t)b * sbytes;
    const EllRec R = ((const EllRec*)B)[0];
    // the stage block as copied: step records, slot words, values (packed
    // to this stage's own nsteps / npad, not to the buffer capacity)
    const int4* steps = (const int4*)(B + 64);
    const uint32_t* src = (const uint32_t*)(B + 64 + 16 * R.nsteps);
    const T* vv = (const T*)(B + 64 + 16 * R.nsteps + al16(W * R.npad * 4));
    const T* sbw = (const T*)(B + o_b) + shift_of(bw, (int64_t)r0 + R.sa);
    const int npad = R.npad;
    const uint32_t gbase = (uint32_t)(r0 + R.sa);  // global row of stage row 0
    T pb[RG], pv[RG][K];
    uint32_t pa[RG][K], pd[RG];
    bool pact[RG], pok[RG];
    auto prefetch = [&](int q) {
      const int4 st4 = steps[q];  // {first_group, ngroups, row_start, nrows}
#pragma unroll
      for (int g = 0; g < RG; ++g) {
        const int gi = warp + g * NW;
        pact[g] = gi < st4.y;
        const int rl = gi * 32 + lane;
        pok[g] = pact[g] && rl < st4.w;
        const int idx = pact[g] ? (st4.x + gi) * 32 + lane : 0;
        const int row = st4.z + (pok[g] ? rl : 0);  // stage-local row
        pb[g] = pok[g] ? sbw[row] : T(0);
        pd[g] = xw + (((gbase + (uint32_t)row) & xmask) << SH);
        uint32_t wd[W];
#pragma unroll
        for (int w = 0; w < W; ++w) wd[w] = src[w * npad + idx];
#pragma unroll
        for (int k2 = 0; k2 < K; ++k2) {
          const uint32_t sl = (k2 & 1) ? (wd[k2 >> 1] >> 16) : (wd[k2 >> 1] & 0xffffu);
          pa[g][k2] = xw + (sl << SH);
          pv[g][k2] = vv[k2 * npad + idx];
        }
      }
    };
    prefetch(0);
    for (int q = 0; q < R.nsteps; ++q) {
#pragma unroll
      for (int g = 0; g < RG; ++g) {
        if (pact[g]) {  // warp-uniform
          T acc = pb[g];
#pragma unroll
          for (int k2 = 0; k2 < K; ++k2) acc -= pv[g][k2] * lds_x(pa[g][k2], T(0));
          if (pok[g]) sts_x(pd[g], acc);
        }
      }
      if (q + 1 < R.nsteps) {
        prefetch(q + 1);
      } else {
        // the producer's bulk store reads this stage's window rows through
        // the async proxy
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      }
      asm volatile("bar.sync 1, %0;" ::"r"(NC) : "memory");  // level barrier (Alg 2 L96)
    }
    if (trace && tid == 0) trace[3 * s + 2] = clock64();
    if (tid == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(&empty[b])) : "memory");
    if (++b == NST) {
      b = 0;
      ph ^= 1u;
    }
  }
}

// ------------- K4' (B200): strand wavefront over a thread-block cluster
// For a narrow-level triangle (the near-serial / level-set role of Alg 7,
// L256, where the levels are too narrow to fill the GPU and each level would
// cost a grid-wide synchronisation), the rows are split into NS = C x W
// STRANDS: contiguous ranges of the ORIGINAL (lower) row index, balanced in
// rows.  L is lower in the original numbering, so a row depends only on rows
// of its own or of a lower strand; strands form a pipeline, and strand s runs
// a few levels behind strand s-1 (the wavefront).  One warp owns a strand
// and walks its rows in level order as GROUPS of <= 32 rows of one level
// (lane = row), with no barrier at all: the level order inside the warp
// replaces Alg 2's level barrier (L96), and a dependency on another strand
// is a shared-memory value that is its own ready flag (the sentinel of the
// sync-free kernels, Alg 3, kept on-chip):
//   * own strand, within XW positions: the warp's private ring window
//     (written by this warp in an earlier group; __syncwarp orders it);
//   * another strand of the cluster: a unique IMPORT slot in this warp's
//     shared memory; the producing lane PUSHES its x there (st.shared::cluster
//     to the consumer CTA, DSMEM, ~200 cycles) right after computing it, and
//     the consumer spins on its own shared memory (~30 cycles), so the
//     cross-SM hop overlaps the producer's lead instead of sitting on the
//     chain;
//   * anything else (window / import capacity overflow): xs in global memory,
//     polled with strong loads (value-as-flag).
// The execution order of the triangle's rows on the device is strand-major,
// group-major (the upload applies that permutation to the plan's device
// indices), so a group is a contiguous range of rows: its b' arrives by TMA
// and its x stores are coalesced.  Per strand the operands stream through a
// ring of NCH chunks (GPC groups each) filled by cp.async.bulk (lane 0) on
// one mbarrier per chunk; the chunk header carries the row range of chunk
// c + NCH, so no control word is read from global memory inside the loop.
//
// Chunk block: int4 {row_lo, row_hi, next_lo, next_hi} (b' rows of this chunk
// and of chunk c + NCH), one int4 {row_start, cnt | flags, boff, -} per group
// (boff: index of the group's first b' value in the chunk's b' window), then
// GPC group blocks {u32 xoff[K][32], u32 soff[32], u32 push[E][32],
// T vals[K][32]}.
//   xoff: BYTE offset in the CTA's x area of the dependency (own-window or
//         import slot; padding: the zero slot at byte 0).  In a group flagged
//         GF_GLOBAL: bit 31 set = execution-order row of xs polled in global
//         memory instead.
//   soff: byte offset of the row's own-window slot (padding lanes: the sink
//         slot at byte 8).
//   push: (cta rank << 24) | byte offset of an import slot of a consumer
//         strand, ~0u = none.
//
// The loop (one warp = one strand) keeps only this on the level chain:
//   __syncwarp -> LDS x_j -> 2 x DFMA -> STS x_i
// (single-warp microbenchmark: ~51 cycles, scripts/microbench/wave_loop.cu).
// Everything else is off it: the operands of group g+2 are loaded while
// group g waits for its x loads, and there is NO readiness test per group
// (the microbenchmark and the SPTRSV_WAVE_EXP ablation measured ~63 cycles
// per group for any vote + branch, wherever it sits).  Instead a strand
// checks readiness once per chunk: the chunk block ends with the import
// slots its groups use for the first time, and chunk_wait polls them (one
// LDS per lane) until none is the sentinel.  Own-strand values were stored
// by this warp before the last __syncwarp; an import slot is written once,
// so a slot that passed its first-use chunk stays valid.  The price is a
// lag of one chunk (GPC levels) per strand boundary of the wavefront.
constexpr int kWaveGF_GLOBAL = 1 << 30, kWaveGF_PUSH = 1 << 29, kWaveCntMask = (1 << 29) - 1;
struct WaveStrand {
  int off16, nchunk, ngroups, row0;  // row0: first execution-order row of the strand
  int lo[4], hi[4];                  // b' row ranges of chunks 0..3 (the prologue loads)
  uint32_t imp_lo, imp_hi;           // byte range of the strand's import slots in its CTA's x area
  int pad[2];
};
struct WaveGeom {
  int W, GPC, NCH, xa_slots;  // warps per CTA, groups per chunk, ring depth, x area slots per CTA
  uint32_t chunk_bytes, bring_bytes, group_bytes, hdr_bytes;
  int imp_per_lane;           // words per lane of a chunk's first-use import list (after its groups)
};

template <typename T>
__host__ __device__ inline uint32_t wave_group_bytes(int K, int E) {
  return 128u * (uint32_t)K + 128u + 128u * (uint32_t)E + 32u * (uint32_t)K * (uint32_t)sizeof(T);
}
__host__ __device__ inline uint32_t wave_hdr_bytes(int GPC) { return 16u + 16u * (uint32_t)GPC; }
template <typename T>
__host__ __device__ inline uint32_t wave_bring_bytes(int GPC) {
  // + 32 rows of slack: padding lanes of a chunk's last group read (and
  // discard) past the window
  return al16((uint32_t)GPC * 32u * (uint32_t)sizeof(T) + 32u) + 32u * (uint32_t)sizeof(T);
}
template <typename T>
__host__ __device__ inline uint32_t wave_smem_bytes(const WaveGeom& g) {
  return al16((uint32_t)g.xa_slots * (uint32_t)sizeof(T)) +
         (uint32_t)(g.W * g.NCH) * (g.chunk_bytes + g.bring_bytes) + (uint32_t)(g.W * g.NCH) * 16u;
}

__device__ __forceinline__ uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// x loads / stores of the wave loop: volatile (never cached or dropped) and
// ordered among themselves, but without a "memory" clobber so the compiler
// may schedule the operand prefetch around them
__device__ __forceinline__ double lds_x_v(uint32_t a, double) {
  double v;
  asm volatile("ld.volatile.shared.f64 %0, [%1];" : "=d"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ float lds_x_v(uint32_t a, float) {
  float v;
  asm volatile("ld.volatile.shared.f32 %0, [%1];" : "=f"(v) : "r"(a));
  return v;
}
// the level-chain x load: a "memory" clobber pins it ahead of the operand
// prefetch that follows it in program order (the prefetch LDS then queue
// behind it in the MIO pipe instead of delaying it)
__device__ __forceinline__ double lds_x_first(uint32_t a, double) {
  double v;
  asm volatile("ld.volatile.shared.f64 %0, [%1];" : "=d"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ float lds_x_first(uint32_t a, float) {
  float v;
  asm volatile("ld.volatile.shared.f32 %0, [%1];" : "=f"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts_x_v(uint32_t a, double v) {
  asm volatile("st.volatile.shared.f64 [%0], %1;" ::"r"(a), "d"(v));
}
__device__ __forceinline__ void sts_x_v(uint32_t a, float v) {
  asm volatile("st.volatile.shared.f32 [%0], %1;" ::"r"(a), "f"(v));
}
__device__ __forceinline__ double ldg_x_v(const double* p) {
  double v;
  asm volatile("ld.relaxed.gpu.global.f64 %0, [%1];" : "=d"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ float ldg_x_v(const float* p) {
  float v;
  asm volatile("ld.relaxed.gpu.global.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ void stg_x_v(double* p, double v) {
  asm volatile("st.relaxed.gpu.global.f64 [%0], %1;" ::"l"(p), "d"(v));
}
__device__ __forceinline__ void stg_x_v(float* p, float v) {
  asm volatile("st.relaxed.gpu.global.f32 [%0], %1;" ::"l"(p), "f"(v));
}
// push x into a consumer strand's import slot (DSMEM), unless p == ~0u
__device__ __forceinline__ void wave_push(uint32_t p, uint32_t xa_s, double v) {
  asm volatile(
      "{\n .reg .pred q;\n .reg .b32 ra;\n setp.ne.u32 q, %0, -1;\n"
      " @q mapa.shared::cluster.u32 ra, %1, %2;\n @q st.relaxed.cluster.shared::cluster.f64 [ra], %3;\n}\n" ::"r"(p),
      "r"(xa_s + (p & 0xffffffu)), "r"(p >> 24), "d"(v)
      : "memory");
}
__device__ __forceinline__ void wave_push(uint32_t p, uint32_t xa_s, float v) {
  asm volatile(
      "{\n .reg .pred q;\n .reg .b32 ra;\n setp.ne.u32 q, %0, -1;\n"
      " @q mapa.shared::cluster.u32 ra, %1, %2;\n @q st.relaxed.cluster.shared::cluster.f32 [ra], %3;\n}\n" ::"r"(p),
      "r"(xa_s + (p & 0xffffffu)), "r"(p >> 24), "f"(v)
      : "memory");
}
// "might be the sentinel": the high word only (exact test in the wait loop)
__device__ __forceinline__ bool maybe_sent(double v) { return __double2hiint(v) == 0x7FF40000; }
__device__ __forceinline__ bool maybe_sent(float v) { return __float_as_uint(v) == 0x7FA00BADu; }

template <typename T, int K, int E>
struct WaveOp {
  uint32_t xo[K], so;
  uint32_t push[E > 0 ? E : 1];
  T v[K];
  T b;
  int row, cnt;  // cnt with the group flags
};

__device__ __forceinline__ void warp_sync_all() { asm volatile("bar.warp.sync -1;" ::: "memory"); }
__device__ __forceinline__ bool vote_any(bool p) {
  uint32_t r;
  asm volatile("{\n .reg .pred q, r;\n setp.ne.u32 q, %1, 0;\n vote.sync.any.pred r, q, -1;\n selp.u32 %0, 1, 0, r;\n}\n"
               : "=r"(r)
               : "r"((uint32_t)p));
  return r != 0;
}

// GPC (groups per chunk, even) is a template parameter so the group loop of
// a chunk is fully unrolled: the operand sets alternate between two register
// sets without copies, the chunk switch happens only at the last group, and
// padding groups (cnt 0: zero-slot operands, sink store, no global store, no
// push) execute as no-ops instead of being branched around.  GLB: some group
// polls xs in global memory (window / import overflow).
__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t parity) {
  uint32_t done;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(done)
      : "r"(smem_addr(bar)), "r"(parity)
      : "memory");
  return done != 0;
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(bar)) : "memory");
}

// Block = W consumer warps (one strand each) + one producer warp that keeps
// every strand's ring of NCH chunks filled by TMA (full / empty mbarriers),
// so a consumer never issues a copy: at a chunk end it only arrives on the
// slot's empty barrier and waits on the next slot's full barrier.
#ifndef SPTRSV_WAVE_EXP
#define SPTRSV_WAVE_EXP 0  // instrumented builds drop parts of the loop to time them (tuning only)
#endif
#ifndef SPTRSV_WAVE_WAIT_NS
#define SPTRSV_WAVE_WAIT_NS 64
#endif
constexpr unsigned kWaveWaitNs = SPTRSV_WAVE_WAIT_NS;
#ifndef SPTRSV_WAVE_GPC_BIG
#define SPTRSV_WAVE_GPC_BIG 12
#endif
constexpr int kWaveGpcBig = SPTRSV_WAVE_GPC_BIG;  // groups per chunk (multiple of 3); 6 when smem is short
#ifndef SPTRSV_WAVE_Q
#define SPTRSV_WAVE_Q 1  // measured on C2: 1 0.2586 ms, 2 0.2597, 3 0.2668
#endif
constexpr int kWaveQ = SPTRSV_WAVE_Q;  // import checks per chunk (divides 6)
template <typename T, int K, int E, int GPC, bool GLB>
__global__ void __launch_bounds__(288, 1)
    tri_wave(const WaveStrand* __restrict__ strands, const char* __restrict__ data, const T* __restrict__ bw, T* __restrict__ xs, WaveGeom g, SolveState st, long long* __restrict__ trace) {
  extern __shared__ __align__(128) unsigned char smem[];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const uint32_t rank = cluster_ctarank();
  T* xa = (T*)smem;
  const uint32_t xa_s = smem_addr(smem);
  unsigned char* ring0 = smem + al16((uint32_t)g.xa_slots * (uint32_t)sizeof(T));
  unsigned char* bring0 = ring0 + (size_t)(g.W * g.NCH) * g.chunk_bytes;
  uint64_t* full0 = (uint64_t*)(bring0 + (size_t)(g.W * g.NCH) * g.bring_bytes);
  uint64_t* empty0 = full0 + g.W * g.NCH;
  // x area: slot 0 zero (padding dependencies), slot 1 sink (padding lanes'
  // stores), the rest the sentinel (import slots read "not ready" until pushed)
  for (int i = tid; i < g.xa_slots; i += blockDim.x) xa[i] = i < 2 ? T(0) : sent<T>();
  if (tid == 0)
    for (int c = 0; c < 2 * g.W * g.NCH; ++c) mbar_init(&full0[c], 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncthreads();
  cluster_sync_all();  // every import area is initialised before any push

  if (warp == g.W) {  // ---------------- producer warp: lane w feeds strand w
    const int w = lane;
    int nch = 0, c = 0, off16 = 0;
    if (w < g.W) {
      const WaveStrand* Sp = strands + rank * g.W + w;
      nch = Sp->nchunk;
      off16 = Sp->off16;
    }
    auto issue = [&](int cc, int lo, int hi) {
      const int slot = cc % g.NCH;
      const Win wb = win(bw, (int64_t)lo, hi - lo);
      uint64_t* fb = &full0[w * g.NCH + slot];
      mbar_expect_tx(fb, g.chunk_bytes + wb.bytes);
      tma_bulk_g2s(ring0 + (size_t)(w * g.NCH + slot) * g.chunk_bytes,
                   data + (size_t)off16 * 16 + (size_t)cc * g.chunk_bytes, g.chunk_bytes, fb);
      tma_bulk_g2s(bring0 + (size_t)(w * g.NCH + slot) * g.bring_bytes, wb.src, wb.bytes, fb);
    };
    if (w < g.W) {
      const WaveStrand* Sp = strands + rank * g.W + w;
      for (; c < g.NCH && c < nch; ++c) issue(c, Sp->lo[c], Sp->hi[c]);
    }
    uint32_t idle = 0;
    while (__any_sync(0xffffffffu, c < nch)) {
      bool did = false;
      if (c < nch) {
        const int slot = c % g.NCH;
        // chunk c reuses the slot of chunk c - NCH: wait for its release; the
        // released block's header carries chunk c's b' row range
        if (mbar_test(&empty0[w * g.NCH + slot], (uint32_t)(c / g.NCH - 1) & 1u)) {
          const int4 hdr = *(const int4*)(ring0 + (size_t)(w * g.NCH + slot) * g.chunk_bytes);
          issue(c, hdr.z, hdr.w);
          ++c;
          did = true;
        }
      }
      if (!__any_sync(0xffffffffu, did)) {
        __nanosleep(20);
        if (++idle > (kWatchdogSpins >> 4)) {
          if (lane == 0) watchdog_trip(st);
          break;
        }
      }
    }
    __syncthreads();
    cluster_sync_all();
    return;
  }

  // ---------------- consumer warps
  const WaveStrand* Sp = strands + rank * g.W + warp;
  const int s_nchunk = Sp->nchunk;
  long long* tr = trace ? trace + (size_t)(rank * g.W + warp) * 1024 : nullptr;
  if (tr && lane == 0) tr[0] = clock64();
  unsigned char* ring = ring0 + (size_t)warp * g.NCH * g.chunk_bytes;
  unsigned char* bring = bring0 + (size_t)warp * g.NCH * g.bring_bytes;
  uint64_t* full = full0 + warp * g.NCH;
  uint64_t* empty = empty0 + warp * g.NCH;
  if (tr && lane == 0) tr[1] = clock64();

  uint32_t spins = 0, npolls = 0;
  auto load_op = [&](const unsigned char* B, const T* bb, int gi, WaveOp<T, K, E>& o) {
    const int4 gh = ((const int4*)(B + 16))[gi];
    const uint32_t* wd = (const uint32_t*)(B + g.hdr_bytes + (uint32_t)gi * g.group_bytes);
    const T* vv = (const T*)(wd + 32 * (K + 1 + E));
#pragma unroll
    for (int k2 = 0; k2 < K; ++k2) o.xo[k2] = wd[k2 * 32 + lane];
    o.so = wd[K * 32 + lane];
#pragma unroll
    for (int e = 0; e < E; ++e) o.push[e] = wd[(K + 1 + e) * 32 + lane];
#pragma unroll
    for (int k2 = 0; k2 < K; ++k2) o.v[k2] = vv[k2 * 32 + lane];
    o.b = bb[gh.z + lane];
    o.row = gh.x + lane;
    o.cnt = gh.y;
  };
  // the level-chain part of one group (cur resident)
  auto solve_op = [&](WaveOp<T, K, E>& cur, auto&& mid) -> T {
    T x[K];
    if (!GLB) {
      // ---- level chain: the x_j loads go first, then the next groups'
      // operand prefetch (mid), which overlaps the load latency.  No
      // readiness test here: own-strand values were stored by this warp
      // before the last __syncwarp and every import of the chunk passed
      // chunk_wait at the chunk's start, so the chain is branch-free
      // (LDS x_j -> 2 DFMA -> STS x_i)
#pragma unroll
      for (int k2 = 0; k2 < K; ++k2) x[k2] = lds_x_first(xa_s + cur.xo[k2], T(0));
      mid();
    } else {
      mid();
#pragma unroll
      for (int k2 = 0; k2 < K; ++k2) {
        const bool glb = cur.xo[k2] & 0x80000000u;
        for (;;) {
          x[k2] = glb ? ldg_x_v(xs + (cur.xo[k2] & 0x7fffffffu)) : lds_x_v(xa_s + cur.xo[k2], T(0));
          if (!is_sent(x[k2])) break;
          ++npolls;
          if (++spins > kWatchdogSpins) {
            watchdog_trip(st);
            x[k2] = T(0);
            break;
          }
        }
      }
    }
    T acc = cur.b;
#pragma unroll
    for (int k2 = 0; k2 < K; ++k2) acc = fma(-cur.v[k2], x[k2], acc);
    return acc;
  };
  auto publish = [&](WaveOp<T, K, E>& cur, T acc) {
    sts_x_v(xa_s + cur.so, acc);
    if (!(SPTRSV_WAVE_EXP & 4)) {
#pragma unroll
      for (int e = 0; e < E; ++e) wave_push(cur.push[e], xa_s, acc);
    }
    if (!(SPTRSV_WAVE_EXP & 2) && lane < (cur.cnt & kWaveCntMask)) stg_x_v(xs + cur.row, acc);
  };

  // three operand sets rotate over the groups (GPC % 3 == 0): group g solves
  // from set g%3 while set (g+1)%3 gets its early poll and set (g+2)%3 its
  // operands -- every load has a whole group of lead before its first use
  WaveOp<T, K, E> op0, op1, op2;
  int slot = 0;
  uint32_t ph = 0;
  const unsigned char* B = ring;
  const T* bb = (const T*)bring;
  const unsigned char* Bn = ring;
  const T* bbn = (const T*)bring;
  int slot_n = 0;
  uint32_t ph_n = 0;
  // readiness of a whole chunk: every import slot its groups read must hold
  // a pushed value (not the sentinel) before the chunk starts.  Imports flow
  // only from lower strands, which never wait on this one, so the strand
  // simply runs a chunk behind its producers; one vote per chunk replaces
  // a branch per group on the level chain
  const uint32_t imp_lo = Sp->imp_lo, imp_hi = Sp->imp_hi;
  // The chunk block ends with the byte offsets of the imports the chunk
  // uses first (padding: the zero slot), imp_per_lane words per lane.
  auto chunk_wait = [&](const unsigned char* Bc, int q) {
    const uint32_t* il = (const uint32_t*)(Bc + g.hdr_bytes + (uint32_t)GPC * g.group_bytes +
                                           (uint32_t)(q * g.imp_per_lane) * 128u);
    uint32_t xo0 = 0;
    if (!GLB && g.imp_per_lane > 0) xo0 = il[lane];
    for (; !GLB && imp_lo != imp_hi;) {
      bool pend = is_sent(lds_x_v(xa_s + xo0, T(0)));
      for (int i = 1; i < g.imp_per_lane; ++i) pend |= is_sent(lds_x_v(xa_s + il[i * 32 + lane], T(0)));
      if (!vote_any(pend)) break;
      ++npolls;
      // back off: a spinning warp's polls compete for the SM's shared-memory
      // pipe with the CTA-mate strand that is doing real work
      __nanosleep(kWaveWaitNs);
      if (++spins > kWatchdogSpins) {
        watchdog_trip(st);
        break;
      }
    }
  };
  if (s_nchunk > 0) {
    mbar_wait(&full[0], 0);
    load_op(B, bb, 0, op0);
    load_op(B, bb, 1, op1);
    chunk_wait(B, 0);
  }
  for (int c = 0; c < s_nchunk; ++c) {
    const bool more = c + 1 < s_nchunk;
#pragma unroll
    for (int gi = 0; gi < GPC; ++gi) {
      WaveOp<T, K, E>& cur = gi % 3 == 0 ? op0 : gi % 3 == 1 ? op1 : op2;
      WaveOp<T, K, E>& n1 = gi % 3 == 0 ? op1 : gi % 3 == 1 ? op2 : op0;
      WaveOp<T, K, E>& n2 = gi % 3 == 0 ? op2 : gi % 3 == 1 ? op0 : op1;
      // imports of the next part of the chunk (the first part was checked
      // when the chunk was opened): GPC / kWaveQ levels of lag per strand
      // boundary instead of GPC, one vote per part
      if (gi > 0 && gi % (GPC / kWaveQ) == 0) chunk_wait(B, gi / (GPC / kWaveQ));
#ifdef SPTRSV_WAVE_TRACE
      if (tr && lane == 0 && c * GPC + gi < 1016) {
        long long gt;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt));
        tr[8 + c * GPC + gi] = gt;
      }
#endif
      const T acc = solve_op(cur, [&]() {
        if (gi + 2 < GPC) {
          load_op(B, bb, gi + 2, n2);
        } else if (more) {
          if (gi + 2 == GPC) {  // open the next chunk two groups ahead
            slot_n = slot + 1 == g.NCH ? 0 : slot + 1;
            ph_n = slot + 1 == g.NCH ? ph ^ 1u : ph;
            mbar_wait(&full[slot_n], ph_n);
            Bn = ring + (size_t)slot_n * g.chunk_bytes;
            bbn = (const T*)(bring + (size_t)slot_n * g.bring_bytes);
          }
          load_op(Bn, bbn, gi + 2 - GPC, n2);
        }
      });
      publish(cur, acc);
      if (gi + 1 == GPC) {  // chunk consumed: release its slot to the producer warp
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[slot]);
        slot = slot_n;
        ph = ph_n;
        B = Bn;
        bb = bbn;
        if (more) chunk_wait(B, 0);
      }
      if (!(SPTRSV_WAVE_EXP & 16)) warp_sync_all();
    }
  }
  if (tr && lane == 0) {
    tr[2] = clock64();
    tr[3] = npolls;
    tr[4] = s_nchunk * GPC;
  }
  __syncthreads();
  cluster_sync_all();  // no CTA leaves while a peer may still push into it
}


// ----------------------------------- K2 on one cluster: level-set, no launches
// Level-set (Alg 2 L88-L98) for a triangle whose levels are narrow but many
// (B200 selector, nrhs == 1): the whole triangle runs in ONE thread-block
// cluster (CS CTAs, one per SM), and Alg 2's barrier between levels (L96) is
// the cluster barrier (barrier.cluster.arrive.release / wait.acquire, ~400
// cycles on-chip) instead of a kernel boundary (~2-3 us) or the sync-free
// kernel's per-dependency polls through L2 (Alg 3; on B200 a level of
// ~10^3 rows ends with the slowest of its detections, ~1 us).  No flags, no
// sentinels, no tickets: after the barrier every x of earlier levels is
// visible, so a row's dependencies are plain loads.
//
// Work of level l = the items [ip[l], ip[l+1]) (exec.cu build_cl_items; the
// tri_sf_mixed item kinds, cut at level boundaries): kind 0 = <= 32
// consecutive rows with <= kSfLong entries, lane per row; kind 3 = one row
// of <= kSfNB entries, warp; kind 1/2 = kSfNB-entry pieces of a longer row
// (partial sums to `part` slots, the last piece adds them in piece order).
// Warp gw of the cluster takes items ip[l] + gw, + NW, ...  Between
// barrier.cluster.arrive and .wait each warp already loads the header,
// indices, values and b' of its first item of the next level (they do not
// depend on x), so after the wait only the x gathers remain on the chain.
template <typename T>
struct ClPre {
  int4 h0, h1;
  int p, e, cnt;
  T s;
  int j[kSfNB / 32];
  T v[kSfNB / 32];
};

template <typename T>
__device__ __forceinline__ void cl_load(ClPre<T>& q, const SfItem* __restrict__ items, int w, int r0,
                                        const int* __restrict__ rp, const int* __restrict__ ci,
                                        const T* __restrict__ val, const T* __restrict__ bw, int lane) {
  constexpr int UW = kSfNB / 32;
  q.h0 = __ldg((const int4*)(items + w));
  q.h1 = __ldg((const int4*)(items + w) + 1);
  if (q.h1.x == 0) {
    const int k = q.h0.x + lane;
    q.p = q.e = 0;
    q.s = T(0);
    if (k < q.h0.y) {
      q.p = __ldg(rp + k);
      q.e = __ldg(rp + k + 1);
      q.s = ldg_nc(bw + r0 + k);
    }
    q.cnt = min(UW, q.e - q.p);
#pragma unroll
    for (int u = 0; u < UW; ++u)
      if (u < q.cnt) {
        q.j[u] = __ldg(ci + q.p + u);
        q.v[u] = ldg_nc(val + q.p + u);
      }
  } else {
    const int ne = q.h0.w - q.h0.z;
    q.s = (q.h1.x != 1 && lane == 0) ? ldg_nc(bw + r0 + q.h0.x) : T(0);
#pragma unroll
    for (int u = 0; u < UW; ++u)
      if (lane + 32 * u < ne) {
        q.j[u] = __ldg(ci + q.h0.z + lane + 32 * u);
        q.v[u] = ldg_nc(val + q.h0.z + lane + 32 * u);
      }
  }
}

template <typename T>
__device__ __forceinline__ bool cl_compute(ClPre<T>& q, int r0, const int* __restrict__ ci,
                                           const T* __restrict__ val, T* __restrict__ xs, T* __restrict__ part,
                                           const SolveState& st, uint32_t& spins, int lane) {
  constexpr int UW = kSfNB / 32;
  if (q.h1.x == 0) {
    if (q.h0.x + lane < q.h0.y) {
      T x[UW];
#pragma unroll
      for (int u = 0; u < UW; ++u)
        if (u < q.cnt) x[u] = xs[q.j[u]];
      T s = q.s;
#pragma unroll
      for (int u = 0; u < UW; ++u)
        if (u < q.cnt) s -= q.v[u] * x[u];
      for (int p = q.p + q.cnt; p < q.e; p += UW) {  // rows longer than UW (<= kSfLong)
        const int cnt = min(UW, q.e - p);
#pragma unroll
        for (int u = 0; u < UW; ++u)
          if (u < cnt) {
            q.j[u] = __ldg(ci + p + u);
            q.v[u] = ldg_nc(val + p + u);
          }
#pragma unroll
        for (int u = 0; u < UW; ++u)
          if (u < cnt) x[u] = xs[q.j[u]];
#pragma unroll
        for (int u = 0; u < UW; ++u)
          if (u < cnt) s -= q.v[u] * x[u];
      }
      xs[r0 + q.h0.x + lane] = s;
    }
    return true;
  }
  const int kind = q.h1.x, ne = q.h0.w - q.h0.z;
  T acc = 0;
  {
    T x[UW];
#pragma unroll
    for (int u = 0; u < UW; ++u)
      if (lane + 32 * u < ne) x[u] = xs[q.j[u]];
#pragma unroll
    for (int u = 0; u < UW; ++u)
      if (lane + 32 * u < ne) acc += q.v[u] * x[u];
  }
  acc = warp_sum(acc);
  bool ok = true;
  if (kind == 2) {  // the earlier pieces' partial sums (same level), 32 at a time, in piece order
    T ps = T(0);
    for (int q0 = q.h1.y; q0 < q.h1.z; q0 += 32) {
      T pv = T(0);
      if (q0 + lane < q.h1.z) {
        pv = ld_strong(part + q0 + lane);
        while (is_sent(pv)) {
          if (wd_giveup(spins, st)) {
            ok = false;
            break;
          }
          pv = ld_strong(part + q0 + lane);
        }
      }
      ps += warp_sum(pv);
    }
    acc += ps;
  }
  if (lane == 0) {
    if (kind == 1)
      st_strong(part + q.h1.y, acc);
    else
      xs[r0 + q.h0.x] = q.s - acc;
  }
  return __all_sync(0xffffffffu, ok);
}

#ifndef SPTRSV_CL_NT
#define SPTRSV_CL_NT 512
#endif
template <typename T>
__global__ void __launch_bounds__(SPTRSV_CL_NT, 1)
    tri_level_cluster(int r0, int nlev, const int* __restrict__ ip, const SfItem* __restrict__ items,
                      const int* __restrict__ rp, const int* __restrict__ ci, const T* __restrict__ val,
                      const T* __restrict__ bw, T* __restrict__ xs, T* __restrict__ part, SolveState st) {
  const int lane = threadIdx.x & 31;
  const int nw = gridDim.x * (blockDim.x >> 5);
  const int gw = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  uint32_t spins = 0;
  bool alive = true;
  ClPre<T> q;
  int i0 = __ldg(ip), i1 = __ldg(ip + 1);
  bool have = gw < i1 - i0;
  if (have) cl_load(q, items, i0 + gw, r0, rp, ci, val, bw, lane);
  for (int l = 0; l < nlev; ++l) {
    const int i2 = l + 2 <= nlev ? __ldg(ip + l + 2) : i1;
    if (have && alive) alive = cl_compute(q, r0, ci, val, xs, part, st, spins, lane);
    for (int w = i0 + gw + nw; w < i1 && alive; w += nw) {
      cl_load(q, items, w, r0, rp, ci, val, bw, lane);
      alive = cl_compute(q, r0, ci, val, xs, part, st, spins, lane);
    }
    __syncwarp();
    asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
    have = i1 + gw < i2;
    if (have) cl_load(q, items, i1 + gw, r0, rp, ci, val, bw, lane);
    __syncwarp();
    asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
    i0 = i1;
    i1 = i2;
  }
}


// ------------------------------ transposed solve from the same plan (f-4, R32)
// A^T x = b with the plan of A.  The plan stores L1 = D^-1 P A P^T (unit
// lower, values scaled by 1/d, R27), so A = P^T D L1 P and
//     A^T x = b  <=>  L1^T z = P b,   x = P^T D^-1 z.
// L1^T is unit UPPER: it is solved over the plan's segments in REVERSE order
// with the PUSH form of the sync-free solve, Alg 3 (L105-L125) as the paper
// states it: a component waits until its in-degree counter (here the number
// of not-yet-solved rows whose L1 row references it, i.e. its column count
// inside the triangle) reaches zero, takes z_i = b'_i, then for every entry
// (i, j) of its L1 row adds -l'_ij z_i into b'_j with atomicAdd and
// decrements in_degree[j] (release after a fence).  A square (rows R, cols C)
// of L1 becomes b'_C -= S^T z_R: every stored row pushes its entries with
// atomics.  The same CSR arrays serve both directions: no second plan, no
// transpose of the matrix.

// b'[k] = b[perm[k]] (no 1/d: it moves to permute-out); counters from cnt0;
// block 0 zeroes the per-segment claim tickets
template <typename T>
__global__ void perm_in_T(int n, const int* __restrict__ perm, const T* __restrict__ b, int64_t stride,
                          T* __restrict__ bw, const int* __restrict__ cnt0, int* __restrict__ cnt,
                          uint32_t* __restrict__ tickets, int nticket) {
  if (blockIdx.x == 0)
    for (int t = threadIdx.x; t < nticket; t += blockDim.x) tickets[t] = 0;
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k < n) {
    bw[k] = b[(int64_t)perm[k] * stride];
    cnt[k] = cnt0[k];
  }
}

// x[perm[k]] = z_k / d_k
template <typename T>
__global__ void perm_out_T(int n, const int* __restrict__ perm, const T* __restrict__ rd, const T* __restrict__ xs,
                           T* __restrict__ x, int64_t stride) {
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k < n) x[(int64_t)perm[k] * stride] = xs[k] * rd[k];
}

// in-degree of the transposed triangle: column counts of its CSR entries
static __global__ void count_cols(int64_t nnz, const int* __restrict__ ci, int* __restrict__ cnt0) {
  for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < nnz; p += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(cnt0 + ci[p], 1);
}

__device__ __forceinline__ int ld_acquire(const int* p) {
  int v;
  asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// Transposed triangle (unit upper L1^T), push form.  Warps claim groups of
// 32 components through a ticket in REVERSE topological order (order[i], or
// local row m-1-i when the device row order is the level order), so every
// component a claimed one waits for was claimed earlier and is running: no
// deadlock under any CTA schedule (the argument of the forward kernel).
// Pushes of one row (entries [a, e), value z): a row of <= kPushShort
// entries is pushed by its own lane; longer rows (supernodal panels, hubs)
// by the whole warp, lanes over the entries, one ready row after another.
// Every lane fences (acq_rel) between its own adds and its own decrements:
// the release pattern of Alg 3's "atomicAdd(left_sum) then atomicSub
// (in_degree)" (L118-L123), without a sequentially consistent fence.
constexpr int kPushShort = 8;
__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }

template <typename T, bool CNT>
__device__ __forceinline__ void push_rows(bool ready, int a, int e, T z, const int* __restrict__ ci,
                                          const T* __restrict__ val, T* __restrict__ bw, int* __restrict__ cnt,
                                          int lane) {
  const bool shortr = ready && e - a <= kPushShort;
  if (shortr)
    for (int p = a; p < e; ++p) atomicAdd(bw + __ldg(ci + p), -ldg_nc(val + p) * z);
  unsigned lm = __ballot_sync(0xffffffffu, ready && !shortr);
  unsigned lm2 = lm;
  while (lm) {
    const int src = __ffs(lm) - 1;
    lm &= lm - 1;
    const int pa = __shfl_sync(0xffffffffu, a, src), pe = __shfl_sync(0xffffffffu, e, src);
    const T pz = __shfl_sync(0xffffffffu, z, src);
    for (int p = pa + lane; p < pe; p += 32) atomicAdd(bw + __ldg(ci + p), -ldg_nc(val + p) * pz);
  }
  if (!CNT) return;
  if (__any_sync(0xffffffffu, ready)) fence_acq_rel_gpu();
  if (shortr)
    for (int p = a; p < e; ++p) atomicSub(cnt + __ldg(ci + p), 1);
  while (lm2) {
    const int src = __ffs(lm2) - 1;
    lm2 &= lm2 - 1;
    const int pa = __shfl_sync(0xffffffffu, a, src), pe = __shfl_sync(0xffffffffu, e, src);
    for (int p = pa + lane; p < pe; p += 32) atomicSub(cnt + __ldg(ci + p), 1);
  }
}

// Transposed triangle (unit upper L1^T), push form.  Warps claim groups of
// 32 components through a ticket in REVERSE topological order (order[i], or
// local row m-1-i when the device row order is the level order), so every
// component a claimed one waits for was claimed earlier and is running: no
// deadlock under any CTA schedule (the argument of the forward kernel).
template <typename T>
__global__ void __launch_bounds__(256) tri_push_T(int r0, int m, const int* __restrict__ order,
                                                  const int* __restrict__ rp, const int* __restrict__ ci,
                                                  const T* __restrict__ val, T* __restrict__ bw, T* __restrict__ xs,
                                                  int* __restrict__ cnt, uint32_t* __restrict__ ticket,
                                                  SolveState st) {
  const int lane = threadIdx.x & 31;
  uint32_t spins = 0;
  for (;;) {
    int base = 0;
    if (lane == 0) base = (int)atomicAdd(ticket, 32u);
    base = __shfl_sync(0xffffffffu, base, 0);
    if (base >= m) break;
    const int i = base + lane;
    bool done = i >= m;
    int q = 0;
    if (!done) q = order ? __ldg(order + i) : m - 1 - i;
    const int r = r0 + q;
    int a = 0, e = 0;
    if (!done) {
      a = __ldg(rp + q);
      e = __ldg(rp + q + 1);
    }
    bool give = false;
    while (!__all_sync(0xffffffffu, done)) {
      const bool ready = !done && ld_acquire(cnt + r) == 0;
      T z = T(0);
      if (ready) {
        z = ld_strong(bw + r);  // every push into b'_r happened before its counter release
        xs[r] = z;
      }
      push_rows<T, true>(ready, a, e, z, ci, val, bw, cnt, lane);
      done = done || ready;
      if (!done && wd_giveup(spins, st)) give = true;
      if (__any_sync(0xffffffffu, give)) break;  // garbage result, DEADLOCK reported
    }
    if (__any_sync(0xffffffffu, give)) break;
  }
}

// Transposed triangle with narrow levels (every level <= kPcMaxW rows, the
// C2 stencil factor's anti-diagonals): ONE CTA walks the levels in reverse
// with a __syncthreads per level (Alg 2's barrier, L96, on-chip), so the
// push of Alg 3 needs no counters.  Positions p = 0 .. m-1 are the claim
// order (reverse level order); a push into a target within XW positions of
// the current level's start goes into a shared-memory ring slot (atomicAdd
// on shared memory), a farther one into b' in global memory (then the
// pushing thread fences before the level's barrier).  A row's value is its
// global b' (initial b' plus far pushes, read a level ahead) plus its ring
// slot.  The next level's rows, row bounds, first kPcE entries and global b'
// are loaded during the current level, so the per-level chain is
// barrier -> LDS ring -> FMA -> shared atomics -> barrier.
constexpr int kPcMaxW = 2048, kPcNT = 1024, kPcR = kPcMaxW / kPcNT, kPcE = 2;
template <typename T>
struct PcRow {
  int q, n;      // local device row, entry count
  T g;           // b' of the row (global part)
  int tp[kPcE];  // claim positions of the first kPcE push targets
  T v[kPcE];
};
// Every load of a position's record is independent of the others (no
// order -> row pointer -> entry chain): the record is laid out by claim
// position at the first transposed solve (k::pc_build), and b' is gathered
// into claim-position order before the kernel (k::pc_gather).
template <typename T>
__device__ __forceinline__ void pc_load(PcRow<T>& R, int p, const int* __restrict__ pq,
                                        const int* __restrict__ ecnt, const int* __restrict__ etp,
                                        const T* __restrict__ ev, const T* __restrict__ gpos) {
  R.q = __ldg(pq + p);
  R.n = __ldg(ecnt + p);
  R.g = ld_strong(gpos + p);
#pragma unroll
  for (int u = 0; u < kPcE; ++u) {
    R.tp[u] = __ldg(etp + (size_t)p * kPcE + u);
    R.v[u] = ldg_nc(ev + (size_t)p * kPcE + u);
  }
}

// claim position of every entry's target: tpos[e] = pos[ci[e] - r0] or m-1-(ci[e]-r0)
static __global__ void pc_tpos(int64_t ne, int r0, int m, const int* __restrict__ ci, const int* __restrict__ pos,
                               int* __restrict__ tpos) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < ne; e += (int64_t)gridDim.x * blockDim.x) {
    const int lj = ci[e] - r0;
    tpos[e] = pos ? pos[lj] : m - 1 - lj;
  }
}

// per claim position p: entry count and the first kPcE (target position, value) pairs
template <typename T>
__global__ void pc_build(int m, const int* __restrict__ pq, const int* __restrict__ rp, const int* __restrict__ tpos,
                         const T* __restrict__ val, int* __restrict__ ecnt, int* __restrict__ etp, T* __restrict__ ev) {
  const int p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= m) return;
  const int q = pq[p], a = rp[q], e = rp[q + 1];
  ecnt[p] = e - a;
#pragma unroll
  for (int u = 0; u < kPcE; ++u) {
    etp[(size_t)p * kPcE + u] = a + u < e ? tpos[a + u] : p;
    ev[(size_t)p * kPcE + u] = a + u < e ? val[a + u] : T(0);
  }
}

// b' of the segment's rows in claim-position order
template <typename T>
__global__ void pc_gather(int m, int r0, const int* __restrict__ pq, const T* __restrict__ bw, T* __restrict__ gpos) {
  const int p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p < m) gpos[p] = bw[r0 + pq[p]];
}

template <typename T>
__global__ void __launch_bounds__(kPcNT, 1)
    tri_pushchain_T(int r0, int nlev, const int* __restrict__ lvs, const int* __restrict__ pq,
                    const int* __restrict__ ecnt, const int* __restrict__ etp, const T* __restrict__ ev,
                    T* __restrict__ gpos, const int* __restrict__ rp, const int* __restrict__ tpos,
                    const T* __restrict__ val, T* __restrict__ xs, int XW) {
  extern __shared__ __align__(16) unsigned char pc_smem[];
  T* ring = (T*)pc_smem;
  const int tid = threadIdx.x;
  for (int i = tid; i < XW; i += kPcNT) ring[i] = T(0);
  PcRow<T> R[kPcR];
  int s = __ldg(lvs), e = __ldg(lvs + 1);
#pragma unroll
  for (int k = 0; k < kPcR; ++k)
    if (s + tid + k * kPcNT < e) pc_load(R[k], s + tid + k * kPcNT, pq, ecnt, etp, ev, gpos);
  __syncthreads();
  const uint32_t xm = (uint32_t)XW - 1;  // XW is a power of two
  for (int l = 0; l < nlev; ++l) {
    const int en = l + 2 <= nlev ? __ldg(lvs + l + 2) : e;
    // next level's records, loaded while this level computes (far pushes
    // into them came from levels <= l - 1, fenced before those levels'
    // barriers: a level is <= XW / 2 rows)
    PcRow<T> Rn[kPcR];
#pragma unroll
    for (int k = 0; k < kPcR; ++k)
      if (e + tid + k * kPcNT < en) pc_load(Rn[k], e + tid + k * kPcNT, pq, ecnt, etp, ev, gpos);
    bool far = false;
#pragma unroll
    for (int k = 0; k < kPcR; ++k) {
      const int p = s + tid + k * kPcNT;
      if (p < e) {
        const T z = R[k].g + ring[(uint32_t)p & xm];
        ring[(uint32_t)p & xm] = T(0);
        xs[r0 + R[k].q] = z;
        const int a = R[k].n > kPcE ? __ldg(rp + R[k].q) : 0;  // long rows: the CSR for the rest
        for (int u = 0; u < R[k].n; ++u) {
          int tp = 0;
          T vv = T(0);
          if (u < kPcE) {
#pragma unroll
            for (int w2 = 0; w2 < kPcE; ++w2)  // run-time index into registers
              if (w2 == u) {
                tp = R[k].tp[w2];
                vv = R[k].v[w2];
              }
          } else {
            tp = __ldg(tpos + a + u);
            vv = ldg_nc(val + a + u);
          }
          if (tp < s + XW) {
            atomicAdd(ring + ((uint32_t)tp & xm), -vv * z);
          } else {
            atomicAdd(gpos + tp, -vv * z);
            far = true;
          }
        }
      }
    }
    if (far) __threadfence();
    __syncthreads();  // this level's pushes are in the ring (and far ones in L2)
#pragma unroll
    for (int k = 0; k < kPcR; ++k) R[k] = Rn[k];
    s = e;
    e = en;
  }
}

// Transposed square: b'_c -= sum_r s'_rc z_r, one lane per stored row (long
// rows pushed by the whole warp)
template <typename T, bool DCSR>
__global__ void sq_push_T(int nzr, int r0, const int* __restrict__ rows, const int* __restrict__ rp,
                          const int* __restrict__ ci, const T* __restrict__ val, const T* __restrict__ xs,
                          T* __restrict__ bw) {
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  const int lane = threadIdx.x & 31;
  if (t - lane >= nzr) return;  // whole warp out of range
  const bool live = t < nzr;
  int a = 0, e = 0;
  T z = T(0);
  if (live) {
    const int r = DCSR ? __ldg(rows + t) : r0 + t;
    z = xs[r];
    a = __ldg(rp + t);
    e = __ldg(rp + t + 1);
  }
  push_rows<T, false>(live && e > a, a, e, z, ci, val, bw, nullptr, lane);
}

}  // namespace k
}  // namespace sptrsv
