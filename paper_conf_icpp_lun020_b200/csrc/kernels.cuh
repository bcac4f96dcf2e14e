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
};

__device__ __forceinline__ void reset_tickets(const SolveState& st, int tid, int nthreads) {
  for (int t = tid; t < st.nticket; t += nthreads) st.tickets[t] = 0;
}

__device__ __forceinline__ void watchdog_trip(const SolveState& st) {
  if (st.error) *(volatile int*)st.error = 1;
}

// ------------------------------------------------------------------ permute
// bw[k] = b[perm[k]] / d_k (as * rd), xs[k] = SENT (if a sync-free triangle
// polls it).  nrhs == 1; stride = ldb for row-major input, 1 otherwise.
template <typename T>
__global__ void perm_in_1(int n, const int* __restrict__ perm, const T* __restrict__ rd, const T* __restrict__ b,
                          int64_t stride, T* __restrict__ bw, T* __restrict__ xs, int fill_sent, SolveState st) {
  if (blockIdx.x == 0) reset_tickets(st, threadIdx.x, blockDim.x);
  int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k < n) {
    bw[k] = b[(int64_t)perm[k] * stride] * rd[k];
    if (fill_sent) xs[k] = sent<T>();
  }
}

// x[perm[k]] = xs[k]
template <typename T>
__global__ void perm_out_1(int n, const int* __restrict__ perm, const T* __restrict__ xs, T* __restrict__ x,
                           int64_t stride) {
  int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k < n) x[(int64_t)perm[k] * stride] = xs[k];
}

// Column-major B (n x nrhs, ldb) -> row-major bw: a 32x32 tile transposed in
// shared memory; reads are coalesced along original rows i, writes are 32
// contiguous RHS values of the permuted row iperm[i].
template <typename T>
__global__ void perm_in_cm(int n, int nrhs, const int* __restrict__ iperm, const T* __restrict__ rd,
                           const T* __restrict__ b, int64_t ldb, T* __restrict__ bw, T* __restrict__ xs,
                           int fill_sent, SolveState st) {
  __shared__ T tile[32][33];
  if (blockIdx.x == 0 && blockIdx.y == 0) reset_tickets(st, threadIdx.y * 32 + threadIdx.x, 256);
  int i0 = blockIdx.x * 32, c0 = blockIdx.y * 32;
  for (int cc = threadIdx.y; cc < 32; cc += 8) {
    int i = i0 + threadIdx.x, c = c0 + cc;
    if (i < n && c < nrhs) tile[cc][threadIdx.x] = b[i + (int64_t)c * ldb];
  }
  __syncthreads();
  for (int ii = threadIdx.y; ii < 32; ii += 8) {
    int i = i0 + ii, c = c0 + threadIdx.x;
    if (i < n && c < nrhs) {
      int k = iperm[i];
      bw[(int64_t)k * nrhs + c] = tile[threadIdx.x][ii] * rd[k];
      if (fill_sent) xs[(int64_t)k * nrhs + c] = sent<T>();
    }
  }
}

template <typename T>
__global__ void perm_out_cm(int n, int nrhs, const int* __restrict__ iperm, const T* __restrict__ xs,
                            T* __restrict__ x, int64_t ldx) {
  __shared__ T tile[32][33];
  int i0 = blockIdx.x * 32, c0 = blockIdx.y * 32;
  for (int ii = threadIdx.y; ii < 32; ii += 8) {
    int i = i0 + ii, c = c0 + threadIdx.x;
    if (i < n && c < nrhs) tile[threadIdx.x][ii] = xs[(int64_t)iperm[i] * nrhs + c];
  }
  __syncthreads();
  for (int cc = threadIdx.y; cc < 32; cc += 8) {
    int i = i0 + threadIdx.x, c = c0 + cc;
    if (i < n && c < nrhs) x[i + (int64_t)c * ldx] = tile[cc][threadIdx.x];
  }
}

// Row-major B (ldb >= nrhs): bw[k*nrhs + c] = b[perm[k]*ldb + c] * rd[k]
template <typename T>
__global__ void perm_in_rm(int n, int nrhs, const int* __restrict__ perm, const T* __restrict__ rd,
                           const T* __restrict__ b, int64_t ldb, T* __restrict__ bw, T* __restrict__ xs,
                           int fill_sent, SolveState st) {
  if (blockIdx.x == 0) reset_tickets(st, threadIdx.x, blockDim.x);
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

// SpMM update for nrhs > 1 (K9): a group of G lanes per row, lanes over the
// RHS columns (RPT per lane per pass), entries of the row sequential.
template <typename T, int G, int RPT, bool DCSR>
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
    for (int p = a; p < e; ++p) {
      T v = ldg_nc(val + p);
      const T* xr = xs + (int64_t)ldg_nc(ci + p) * nrhs + c0 + lane;
#pragma unroll
      for (int t = 0; t < RPT; ++t)
        if (c0 + lane + G * t < nrhs) acc[t] += v * ldg_nc(xr + G * t);
    }
    T* br = bw + (int64_t)r * nrhs + c0 + lane;
#pragma unroll
    for (int t = 0; t < RPT; ++t)
      if (c0 + lane + G * t < nrhs) br[G * t] -= acc[t];
  }
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

template <typename T, int G, int RPT>
__device__ __forceinline__ void row_multi_solve(int r, int a, int e, const int* __restrict__ ci,
                                                const T* __restrict__ val, const T* __restrict__ bw,
                                                T* __restrict__ xs, int nrhs, int lane) {
  for (int c0 = 0; c0 < nrhs; c0 += G * RPT) {
    T acc[RPT];
#pragma unroll
    for (int t = 0; t < RPT; ++t)
      acc[t] = (c0 + lane + G * t < nrhs) ? bw[(int64_t)r * nrhs + c0 + lane + G * t] : T(0);
    for (int p = a; p < e; ++p) {
      T v = ldg_nc(val + p);
      const T* xr = xs + (int64_t)ldg_nc(ci + p) * nrhs + c0 + lane;
#pragma unroll
      for (int t = 0; t < RPT; ++t)
        if (c0 + lane + G * t < nrhs) acc[t] -= v * xr[G * t];
    }
    T* xo = xs + (int64_t)r * nrhs + c0 + lane;
#pragma unroll
    for (int t = 0; t < RPT; ++t)
      if (c0 + lane + G * t < nrhs) xo[G * t] = acc[t];
  }
}

template <typename T, int G, int RPT>
__global__ void tri_level_multi(int ra, int rb, int r0, const int* __restrict__ rp, const int* __restrict__ ci,
                                const T* __restrict__ val, const T* __restrict__ bw, T* __restrict__ xs,
                                int nrhs) {
  int r = ra + (blockIdx.x * blockDim.x + threadIdx.x) / G, lane = threadIdx.x % G;
  if (r >= rb) return;
  row_multi_solve<T, G, RPT>(r, rp[r - r0], rp[r - r0 + 1], ci, val, bw, xs, nrhs, lane);
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

template <typename T, int G, int RPT>
__global__ void __launch_bounds__(1024) tri_chain_multi(int r0, int nlev, const int* __restrict__ lp,
                                                        const int* __restrict__ rp, const int* __restrict__ ci,
                                                        const T* __restrict__ val, const T* __restrict__ bw,
                                                        T* __restrict__ xs, int nrhs) {
  const int grp = threadIdx.x / G, ng = blockDim.x / G, lane = threadIdx.x % G;
  for (int l = 0; l < nlev; ++l) {
    int ra = r0 + lp[l], rb = r0 + lp[l + 1];
    for (int r = ra + grp; r < rb; r += ng)
      row_multi_solve<T, G, RPT>(r, rp[r - r0], rp[r - r0 + 1], ci, val, bw, xs, nrhs, lane);
    __syncthreads();
  }
}

// ------------------------------------------------ K3: sync-free (multi-CTA)
// Sync-free SpTRSV (Alg 3) for sm_100a in its pull (CSR) form.
// Components are claimed from a per-segment ticket in row order, so every
// dependency of a claimed row was claimed earlier by a running warp: no
// deadlock whatever the CTA scheduling.  A dependency is "satisfied" (the
// in-degree test of Alg 3) when its x_j is no longer the sentinel.
//
// Thread-per-component: a warp claims 32 consecutive rows; each lane
// consumes its dependencies in batches of U independent loads, stopping at
// the first unsolved one and retrying on the next pass (non-blocking, so a
// lane never blocks a lower lane of its own warp that it depends on).
template <typename T, int U>
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
      p = rp[k];
      e = rp[k + 1];
      s = bw[r];
    }
    uint32_t spins = 0;
    while (__any_sync(0xffffffffu, !done)) {
      if (!done) {
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
          progress = took == cnt;
        }
        if (p == e) {
          st_strong(xs + r, s);
          done = true;
        } else if (++spins > kWatchdogSpins) {
          watchdog_trip(st);
          p = e;  // give up: garbage result, reported to the host
        }
      }
    }
  }
}

// Warp-per-component (long rows): lanes stride the dependencies, U per lane
// per batch, all loads of a batch in flight together; a lane spins only on
// dependencies, which all precede the row in ticket order.
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
            if (++spins > kWatchdogSpins) {
              watchdog_trip(st);
              break;
            }
            x[u] = ld_strong(xs + j[u]);
          }
          s += v[u] * x[u];
        }
      }
    }
    s = warp_sum(s);
    if (lane == 0) st_strong(xs + r, bw[r] - s);
  }
}

// Multi-RHS sync-free: a group of G lanes per component, lanes over RHS
// columns; each lane polls exactly the x_j values it consumes.
template <typename T, int G, int RPT>
__global__ void __launch_bounds__(256) tri_syncfree_multi(int r0, int m, const int* __restrict__ rp,
                                                          const int* __restrict__ ci, const T* __restrict__ val,
                                                          const T* __restrict__ bw, T* __restrict__ xs,
                                                          SolveState st, int slot, int nrhs) {
  const int lane = threadIdx.x % G;
  const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << ((threadIdx.x & 31) / G * G));
  uint32_t* ticket = st.tickets + slot;
  while (true) {
    int k = 0;
    if (lane == 0) k = (int)atomicAdd(ticket, 1u);
    k = __shfl_sync(gmask, k, 0, G);
    if (k >= m) break;
    const int r = r0 + k;
    const int a = rp[k], e = rp[k + 1];
    for (int c0 = 0; c0 < nrhs; c0 += G * RPT) {
      T acc[RPT];
#pragma unroll
      for (int t = 0; t < RPT; ++t)
        acc[t] = (c0 + lane + G * t < nrhs) ? bw[(int64_t)r * nrhs + c0 + lane + G * t] : T(0);
      for (int p = a; p < e; ++p) {
        const int j = ldg_nc(ci + p);
        const T v = ldg_nc(val + p);
        const T* xr = xs + (int64_t)j * nrhs + c0 + lane;
        T x[RPT];
#pragma unroll
        for (int t = 0; t < RPT; ++t)
          if (c0 + lane + G * t < nrhs) x[t] = ld_strong(xr + G * t);
#pragma unroll
        for (int t = 0; t < RPT; ++t)
          if (c0 + lane + G * t < nrhs) {
            uint32_t spins = 0;
            while (is_sent(x[t])) {
              if (++spins > kWatchdogSpins) {
                watchdog_trip(st);
                break;
              }
              x[t] = ld_strong(xr + G * t);
            }
            acc[t] -= v * x[t];
          }
      }
      T* xo = xs + (int64_t)r * nrhs + c0 + lane;
#pragma unroll
      for (int t = 0; t < RPT; ++t)
        if (c0 + lane + G * t < nrhs) st_strong(xo + G * t, acc[t]);
    }
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
// analysis), each stage ships an ELL block instead of CSR: for slot k and
// stage row i, the dependency's WINDOW SLOT (j mod XW; XW = a zero slot for
// padding) and its value, column-major so lanes read consecutive words.  A
// row is then K x {LDS slot, LDS value, LDS x, DFMA}: no row pointers, no
// branches, no modulo on the dependency chain.
struct EllRec {
  int sa, sb, l0, nl, off16, npad, pad0, pad1;  // off16: stage block offset in 16-byte units
};

template <typename T>
__host__ __device__ inline uint32_t ell_stage_bytes(int K, int RMAX) {
  const int npad = (RMAX + 3) & ~3;
  return 64 + al16(K * npad * 4) + al16(K * npad * (uint32_t)sizeof(T)) + al16((RMAX + 4) * (uint32_t)sizeof(T)) +
         al16((RMAX + 8) * 4);
}

template <typename T, int K, int RPT>
__global__ void __launch_bounds__(1024, 1)
    tri_chain_ell(int r0, int nstage, const EllRec* __restrict__ recs, const int* __restrict__ lp,
                  const char* __restrict__ ell, const T* __restrict__ bw, T* __restrict__ xs, int NST, int RMAX,
                  int XW, long long* __restrict__ trace) {
  extern __shared__ __align__(128) unsigned char smem[];
  const int tid = threadIdx.x;
  const int NC = blockDim.x - 32;
  const int xmask = XW - 1;
  const int npad_max = (RMAX + 3) & ~3;
  const uint32_t cap_idx = al16(K * npad_max * 4), cap_val = al16(K * npad_max * (uint32_t)sizeof(T));
  const uint32_t cap_b = al16((RMAX + 4) * (uint32_t)sizeof(T));
  const uint32_t sbytes = ell_stage_bytes<T>(K, RMAX);
  T* xw = (T*)(smem + NST * sbytes);  // XW slots + one zero slot
  uint64_t* full = (uint64_t*)(smem + NST * sbytes + al16((XW + 2) * (uint32_t)sizeof(T)));
  uint64_t* empty = full + NST;
  if (tid == 0) {
    for (int b = 0; b < NST; ++b) {
      mbar_init(&full[b], 1);
      mbar_init(&empty[b], 1);
    }
    xw[XW] = T(0);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto base_of = [&](int b) { return smem + (size_t)b * sbytes; };

  if (tid >= NC) {  // ---------------- producer warp
    if (tid == NC) {
      int b = 0;
      uint32_t ph = 0;
      for (int s = 0; s < nstage; ++s) {
        unsigned char* B = base_of(b);
        EllRec R;
        if (s < NST) {
          R = recs[2 * s];
        } else {
          mbar_wait(&empty[b], ph ^ 1u);
          R = ((const EllRec*)B)[1];
        }
        const int n = R.sb - R.sa;
        const uint32_t blk_idx = al16(K * R.npad * 4), blk_val = al16(K * R.npad * (uint32_t)sizeof(T));
        Win wb = win(bw, (int64_t)r0 + R.sa, n);
        Win wl = win(lp, R.l0, R.nl);
        uint32_t tot = 64 + blk_idx + blk_val + wb.bytes + wl.bytes;
        mbar_expect_tx(&full[b], tot);
        tma_bulk_g2s(B, recs + 2 * s, 64, &full[b]);
        const char* src = ell + (size_t)R.off16 * 16;
        tma_bulk_g2s(B + 64, src, blk_idx, &full[b]);
        tma_bulk_g2s(B + 64 + cap_idx, src + blk_idx, blk_val, &full[b]);
        tma_bulk_g2s(B + 64 + cap_idx + cap_val, wb.src, wb.bytes, &full[b]);
        tma_bulk_g2s(B + 64 + cap_idx + cap_val + cap_b, wl.src, wl.bytes, &full[b]);
        if (++b == NST) {
          b = 0;
          ph ^= 1u;
        }
      }
    }
    return;
  }

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
    unsigned char* B = base_of(b);
    const EllRec R = ((const EllRec*)B)[0];
    const int npad = R.npad;
    const int* s_idx = (const int*)(B + 64);
    const T* s_val = (const T*)(B + 64 + cap_idx);
    const T* s_b = (const T*)(B + 64 + cap_idx + cap_val) + shift_of(bw, (int64_t)r0 + R.sa);
    const int* s_lp = (const int*)(B + 64 + cap_idx + cap_val + cap_b) + shift_of(lp, R.l0);
    // Software pipeline across levels: this thread's rows of level li+1
    // (rows la + tid + q*NC, q < RPT) -- their b, slots and values, none of
    // which depend on x -- are loaded before the barrier that ends level li,
    // so after it only ld.shared x -> DFMA -> store remains on the dependency
    // chain.  Branch-free: a row slot past the level end loads row 0 of the
    // stage and is neutralised (slot = the zero slot, value 0, b 0); only the
    // stores are predicated.
    const int nrow = R.sb - R.sa;
    int la = max(s_lp[0], R.sa) - R.sa, lb = min(s_lp[1], R.sb) - R.sa;  // stage-local
    T pb[RPT], pv[RPT][K];
    int ps[RPT][K];
    auto prefetch = [&](int la_, int lb_) {
#pragma unroll
      for (int q = 0; q < RPT; ++q) {
        const int i = la_ + tid + q * NC;
        const bool ok = i < lb_;
        const int ic = ok ? i : 0;
        pb[q] = ok ? s_b[ic] : T(0);
#pragma unroll
        for (int k = 0; k < K; ++k) {
          const int sl = s_idx[k * npad + ic];
          const T v = s_val[k * npad + ic];
          ps[q][k] = ok ? sl : XW;
          pv[q][k] = ok ? v : T(0);
        }
      }
    };
    prefetch(la, lb);
    T* const xs_stage = xs + r0 + R.sa;
    const int sa_mask = R.sa;  // row r = sa + i; window slot (sa + i) & xmask
    for (int li = 0; li + 1 < R.nl; ++li) {
#pragma unroll
      for (int q = 0; q < RPT; ++q) {  // operands already in registers
        T acc = pb[q];
#pragma unroll
        for (int k = 0; k < K; ++k) acc -= pv[q][k] * xw[ps[q][k]];
        const int i = la + tid + q * NC;
        if (i < lb) {
          xw[(sa_mask + i) & xmask] = acc;
          xs_stage[i] = acc;
        }
      }
      if (lb - la > RPT * NC) {  // warp-uniform: a level wider than NC * RPT rows
        for (int i = la + tid + RPT * NC; i < lb; i += NC) {
          T a2 = s_b[i];
#pragma unroll
          for (int k = 0; k < K; ++k) a2 -= s_val[k * npad + i] * xw[s_idx[k * npad + i]];
          xw[(sa_mask + i) & xmask] = a2;
          xs_stage[i] = a2;
        }
      }
      if (li + 2 < R.nl) {
        la = max(s_lp[li + 1] - R.sa, 0);
        lb = min(s_lp[li + 2] - R.sa, nrow);
        prefetch(la, lb);
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

}  // namespace k
}  // namespace sptrsv
