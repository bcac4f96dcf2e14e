// sm_100a kernels of the recursive-block SpTRSV (Alg 7).
//
// Data layout: every solve works on ONE permuted vector
// w = P b (row-major n x nrhs: the nrhs values of a component are contiguous).
// Squares subtract A x from the rows of w they cover (b_si <- b_si - A x, the
// paper's SpMV "updating b", L146/L164), triangles overwrite their rows of w
// with x (b'_i is read once by its own row and replaced by x_i), so w doubles
// as left_sum of Alg 1/Alg 3 and no separate b' / x' / left_sum arrays exist.
//
// Memory-ordering rules used below (verified in SASS):
//   * st.release.gpu  -> MEMBAR.ALL.GPU + STG.STRONG.GPU (publish x, then flag)
//   * ld.relaxed.gpu  -> LDG.STRONG.GPU (served by L2, never a stale L1 line)
//   * ld.acquire.gpu would add CCTL.IVALL (whole-L1 invalidate) per poll, so
//     the spin uses relaxed strong loads and reads x with strong loads after
//     the flag is observed (control-dependent, issued after the flag returns).
#pragma once
#include <cstdint>

namespace sptrsv {
namespace k {

constexpr uint32_t kWatchdogSpins = 1u << 24;  // ~ seconds of polling

__device__ __forceinline__ int ld_flag(const int* p) {
  int v;
  asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_flag_release(int* p, int v) {
  asm volatile("st.release.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
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
  uint32_t* epoch;    // device word, bumped by permute-in
  uint32_t* tickets;  // per-segment row-claim counters, zeroed by permute-in
  int nticket;
  int* error;         // mapped host word (watchdog)
};

// ------------------------------------------------------------------ permute
// w[k] = b[perm[k]]  (nrhs == 1; stride = ldb for row-major input, 1 otherwise)
template <typename T>
__global__ void perm_in_1(int n, const int* __restrict__ perm, const T* __restrict__ b, int64_t stride,
                          T* __restrict__ w, SolveState st) {
  if (blockIdx.x == 0) {
    for (int t = threadIdx.x; t < st.nticket; t += blockDim.x) st.tickets[t] = 0;
    if (threadIdx.x == 0) *st.epoch += 1u;
  }
  int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k < n) w[k] = b[(int64_t)perm[k] * stride];
}

// x[perm[k]] = w[k]
template <typename T>
__global__ void perm_out_1(int n, const int* __restrict__ perm, const T* __restrict__ w, T* __restrict__ x,
                           int64_t stride) {
  int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k < n) x[(int64_t)perm[k] * stride] = w[k];
}

// Column-major B (n x nrhs, ldb) -> row-major w: a 32x32 tile transposed in
// shared memory; reads are coalesced along original rows i, writes are
// 32 contiguous RHS values of the permuted row iperm[i].
template <typename T>
__global__ void perm_in_cm(int n, int nrhs, const int* __restrict__ iperm, const T* __restrict__ b, int64_t ldb,
                           T* __restrict__ w, SolveState st) {
  __shared__ T tile[32][33];
  if (blockIdx.x == 0 && blockIdx.y == 0) {
    int t = threadIdx.y * 32 + threadIdx.x;
    for (; t < st.nticket; t += 256) st.tickets[t] = 0;
    if (threadIdx.x == 0 && threadIdx.y == 0) *st.epoch += 1u;
  }
  int i0 = blockIdx.x * 32, c0 = blockIdx.y * 32;
  for (int cc = threadIdx.y; cc < 32; cc += 8) {
    int i = i0 + threadIdx.x, c = c0 + cc;
    if (i < n && c < nrhs) tile[cc][threadIdx.x] = b[i + (int64_t)c * ldb];
  }
  __syncthreads();
  for (int ii = threadIdx.y; ii < 32; ii += 8) {
    int i = i0 + ii, c = c0 + threadIdx.x;
    if (i < n && c < nrhs) w[(int64_t)iperm[i] * nrhs + c] = tile[threadIdx.x][ii];
  }
}

template <typename T>
__global__ void perm_out_cm(int n, int nrhs, const int* __restrict__ iperm, const T* __restrict__ w,
                            T* __restrict__ x, int64_t ldx) {
  __shared__ T tile[32][33];
  int i0 = blockIdx.x * 32, c0 = blockIdx.y * 32;
  for (int ii = threadIdx.y; ii < 32; ii += 8) {
    int i = i0 + ii, c = c0 + threadIdx.x;
    if (i < n && c < nrhs) tile[threadIdx.x][ii] = w[(int64_t)iperm[i] * nrhs + c];
  }
  __syncthreads();
  for (int cc = threadIdx.y; cc < 32; cc += 8) {
    int i = i0 + threadIdx.x, c = c0 + cc;
    if (i < n && c < nrhs) x[i + (int64_t)c * ldx] = tile[cc][threadIdx.x];
  }
}

// Row-major B (ldb >= nrhs): w[k*nrhs + c] = b[perm[k]*ldb + c]
template <typename T>
__global__ void perm_in_rm(int n, int nrhs, const int* __restrict__ perm, const T* __restrict__ b, int64_t ldb,
                           T* __restrict__ w, SolveState st) {
  if (blockIdx.x == 0) {
    for (int t = threadIdx.x; t < st.nticket; t += blockDim.x) st.tickets[t] = 0;
    if (threadIdx.x == 0) *st.epoch += 1u;
  }
  int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e < (int64_t)n * nrhs) {
    int k = (int)(e / nrhs), c = (int)(e % nrhs);
    w[e] = b[(int64_t)perm[k] * ldb + c];
  }
}

template <typename T>
__global__ void perm_out_rm(int n, int nrhs, const int* __restrict__ perm, const T* __restrict__ w,
                            T* __restrict__ x, int64_t ldx) {
  int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e < (int64_t)n * nrhs) {
    int k = (int)(e / nrhs), c = (int)(e % nrhs);
    x[(int64_t)perm[k] * ldx + c] = w[e];
  }
}

// ------------------------------------------------------- K1: diagonal triangle
// SPTRSV-COMPLETELYPARALLEL (L247 structure 1, Alg 7): x_i = b_i / d_i
template <typename T>
__global__ void tri_diag(int r0, int m, int nrhs, const T* __restrict__ diag, T* __restrict__ w) {
  int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e < (int64_t)m * nrhs) {
    int r = r0 + (int)(e / nrhs);
    w[(int64_t)r0 * nrhs + e] = w[(int64_t)r0 * nrhs + e] / diag[r];
  }
}

// ------------------------------------------ square blocks: b_rows -= A x_cols
// SPMV-SCALAR-CSR / -DCSR (L249-L250, Alg 7): one thread per row.
// nrhs == 1.  x_cols and the rows written are disjoint ranges of w, so x is
// read through the read-only path.
template <typename T, bool DCSR>
__global__ void sq_scalar_1(int nzr, int r0, const int* __restrict__ rows, const int* __restrict__ rp,
                            const int* __restrict__ ci, const T* __restrict__ val, T* __restrict__ w) {
  int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= nzr) return;
  int r = DCSR ? rows[t] : r0 + t;
  int a = rp[t], e = rp[t + 1];
  T s = 0;
  for (int p = a; p < e; ++p) s += ldg_nc(val + p) * ldg_nc(w + ldg_nc(ci + p));
  w[r] -= s;
}

// SPMV-VECTOR-CSR / -DCSR (L249-L250, Alg 7): a warp per row.
template <typename T, bool DCSR>
__global__ void sq_vector_1(int nzr, int r0, const int* __restrict__ rows, const int* __restrict__ rp,
                            const int* __restrict__ ci, const T* __restrict__ val, T* __restrict__ w) {
  int wid = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (wid >= nzr) return;
  int a = rp[wid], e = rp[wid + 1];
  T s = 0;
  for (int p = a + lane; p < e; p += 32) s += ldg_nc(val + p) * ldg_nc(w + ldg_nc(ci + p));
  s = warp_sum(s);
  if (lane == 0) {
    int r = DCSR ? rows[wid] : r0 + wid;
    w[r] -= s;
  }
}

// SpMM update for nrhs > 1 (K9): a group of G lanes per row, lanes over the
// RHS columns (RPT per lane per pass), entries of the row sequential.
template <typename T, int G, int RPT, bool DCSR>
__global__ void sq_multi(int nzr, int r0, const int* __restrict__ rows, const int* __restrict__ rp,
                         const int* __restrict__ ci, const T* __restrict__ val, T* __restrict__ w, int nrhs) {
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
      const T* xr = w + (int64_t)ldg_nc(ci + p) * nrhs + c0 + lane;
#pragma unroll
      for (int t = 0; t < RPT; ++t)
        if (c0 + lane + G * t < nrhs) acc[t] += v * ldg_nc(xr + G * t);
    }
    T* wr = w + (int64_t)r * nrhs + c0 + lane;
#pragma unroll
    for (int t = 0; t < RPT; ++t)
      if (c0 + lane + G * t < nrhs) wr[G * t] -= acc[t];
  }
}

// ------------------------------------------------- K2: one level of a triangle
// SPTRSV-LEVEL-SET (Alg 2 L88-L98; L247 "a thread or a 32-thread warp"): after
// the level reorder every level is a contiguous row range [ra, rb).  One
// launch per level; the launch boundary is the barrier of Alg 2 L96.
template <typename T, bool WARP>
__global__ void tri_level_1(int ra, int rb, int r0, const int* __restrict__ rp, const int* __restrict__ ci,
                            const T* __restrict__ val, const T* __restrict__ diag, T* __restrict__ w) {
  int r;
  int lane = threadIdx.x & 31;
  if (WARP) {
    r = ra + ((blockIdx.x * blockDim.x + threadIdx.x) >> 5);
  } else {
    r = ra + blockIdx.x * blockDim.x + threadIdx.x;
  }
  if (r >= rb) return;
  int a = rp[r - r0], e = rp[r - r0 + 1];
  T s = 0;
  if (WARP) {
    for (int p = a + lane; p < e; p += 32) s += ldg_nc(val + p) * w[ldg_nc(ci + p)];
    s = warp_sum(s);
    if (lane == 0) w[r] = (w[r] - s) / diag[r];
  } else {
    for (int p = a; p < e; ++p) s += ldg_nc(val + p) * w[ldg_nc(ci + p)];
    w[r] = (w[r] - s) / diag[r];
  }
}

template <typename T, int G, int RPT>
__device__ __forceinline__ void row_multi_solve(int r, int a, int e, const int* __restrict__ ci,
                                                const T* __restrict__ val, T d, T* __restrict__ w, int nrhs,
                                                int lane) {
  for (int c0 = 0; c0 < nrhs; c0 += G * RPT) {
    T acc[RPT];
#pragma unroll
    for (int t = 0; t < RPT; ++t) acc[t] = 0;
    for (int p = a; p < e; ++p) {
      T v = ldg_nc(val + p);
      const T* xr = w + (int64_t)ldg_nc(ci + p) * nrhs + c0 + lane;
#pragma unroll
      for (int t = 0; t < RPT; ++t)
        if (c0 + lane + G * t < nrhs) acc[t] += v * xr[G * t];
    }
    T* wr = w + (int64_t)r * nrhs + c0 + lane;
#pragma unroll
    for (int t = 0; t < RPT; ++t)
      if (c0 + lane + G * t < nrhs) wr[G * t] = (wr[G * t] - acc[t]) / d;
  }
}

template <typename T, int G, int RPT>
__global__ void tri_level_multi(int ra, int rb, int r0, const int* __restrict__ rp, const int* __restrict__ ci,
                                const T* __restrict__ val, const T* __restrict__ diag, T* __restrict__ w,
                                int nrhs) {
  int r = ra + (blockIdx.x * blockDim.x + threadIdx.x) / G, lane = threadIdx.x % G;
  if (r >= rb) return;
  row_multi_solve<T, G, RPT>(r, rp[r - r0], rp[r - r0 + 1], ci, val, diag[r], w, nrhs, lane);
}

// ---------------------------------------- K4: single-CTA level chain (near-serial)
// The cuSPARSE role of Alg 7 (L256, L272-L273) and, under the B200 selector,
// every triangle whose levels are narrow: one CTA walks the levels in order
// and separates them with bar.sync (~tens of cycles) instead of a kernel
// launch or cross-SM flags.  Rows written in earlier levels are read with
// plain (L1-coherent within the SM) loads -- NOT the non-coherent path.
template <typename T, bool WARP>
__global__ void __launch_bounds__(1024) tri_chain_1(int r0, int nlev, const int* __restrict__ lp,
                                                    const int* __restrict__ rp, const int* __restrict__ ci,
                                                    const T* __restrict__ val, const T* __restrict__ diag,
                                                    T* __restrict__ w) {
  const int tid = threadIdx.x, nt = blockDim.x;
  const int lane = tid & 31, wid = tid >> 5, nw = nt >> 5;
  for (int l = 0; l < nlev; ++l) {
    int ra = r0 + lp[l], rb = r0 + lp[l + 1];
    if (WARP) {
      for (int r = ra + wid; r < rb; r += nw) {
        int a = rp[r - r0], e = rp[r - r0 + 1];
        T s = 0;
        for (int p = a + lane; p < e; p += 32) s += ldg_nc(val + p) * w[ldg_nc(ci + p)];
        s = warp_sum(s);
        if (lane == 0) w[r] = (w[r] - s) / diag[r];
      }
    } else {
      for (int r = ra + tid; r < rb; r += nt) {
        int a = rp[r - r0], e = rp[r - r0 + 1];
        T s = 0;
        for (int p = a; p < e; ++p) s += ldg_nc(val + p) * w[ldg_nc(ci + p)];
        w[r] = (w[r] - s) / diag[r];
      }
    }
    __syncthreads();
  }
}

template <typename T, int G, int RPT>
__global__ void __launch_bounds__(1024) tri_chain_multi(int r0, int nlev, const int* __restrict__ lp,
                                                        const int* __restrict__ rp, const int* __restrict__ ci,
                                                        const T* __restrict__ val, const T* __restrict__ diag,
                                                        T* __restrict__ w, int nrhs) {
  const int grp = threadIdx.x / G, ng = blockDim.x / G, lane = threadIdx.x % G;
  for (int l = 0; l < nlev; ++l) {
    int ra = r0 + lp[l], rb = r0 + lp[l + 1];
    for (int r = ra + grp; r < rb; r += ng)
      row_multi_solve<T, G, RPT>(r, rp[r - r0], rp[r - r0 + 1], ci, val, diag[r], w, nrhs, lane);
    __syncthreads();
  }
}

// ------------------------------------------------ K3: sync-free (multi-CTA)
// Sync-free SpTRSV (Alg 3) for sm_100a in its pull (CSR) form:
// a component is claimed from a per-segment ticket in row order (so every
// dependency of a claimed row was claimed earlier by a running warp: no
// deadlock regardless of CTA scheduling), waits until each dependency's ready
// flag equals this solve's epoch (the in-degree test of Alg 3, with the
// counter replaced by one flag per component: no reset, no atomics on the
// hot path), computes x_i and publishes it with a release store.
//
// Thread-per-component variant: a warp claims 32 consecutive rows; each lane
// advances through its row's dependencies as they become ready (non-blocking,
// so a lane never blocks a lower lane of its own warp that it depends on).
template <typename T>
__global__ void __launch_bounds__(256) tri_syncfree_thread(int r0, int m, const int* __restrict__ rp,
                                                           const int* __restrict__ ci,
                                                           const T* __restrict__ val, const T* __restrict__ diag,
                                                           T* __restrict__ w, int* __restrict__ flags,
                                                           SolveState st, int slot) {
  const int lane = threadIdx.x & 31;
  const int epoch = (int)*((volatile uint32_t*)st.epoch);
  uint32_t* ticket = st.tickets + slot;
  while (true) {
    int base = 0;
    if (lane == 0) base = (int)atomicAdd(ticket, 32u);
    base = __shfl_sync(0xffffffffu, base, 0);
    if (base >= m) break;
    int k = base + lane;
    bool done = k >= m;
    int r = r0 + k;
    int p = 0, e = 0;
    T s = 0;
    if (!done) {
      p = rp[k];
      e = rp[k + 1];
    }
    uint32_t spins = 0;
    while (__any_sync(0xffffffffu, !done)) {
      if (!done) {
        while (p < e) {
          int j = ldg_nc(ci + p);
          if (ld_flag(flags + j) != epoch) break;
          s += ldg_nc(val + p) * ld_strong(w + j);
          ++p;
        }
        if (p == e) {
          T x = (w[r] - s) / diag[r];
          w[r] = x;
          st_flag_release(flags + r, epoch);
          done = true;
        } else if (++spins > kWatchdogSpins) {
          if (st.error) *(volatile int*)st.error = 1;
          p = e;  // give up: garbage result, flagged to the host
        }
      }
    }
  }
}

// Warp-per-component variant (long rows): lanes stride the dependencies and
// each spins on its own; the dependencies all precede the row in ticket order.
template <typename T>
__global__ void __launch_bounds__(256) tri_syncfree_warp(int r0, int m, const int* __restrict__ rp,
                                                         const int* __restrict__ ci, const T* __restrict__ val,
                                                         const T* __restrict__ diag, T* __restrict__ w,
                                                         int* __restrict__ flags, SolveState st, int slot) {
  const int lane = threadIdx.x & 31;
  const int epoch = (int)*((volatile uint32_t*)st.epoch);
  uint32_t* ticket = st.tickets + slot;
  while (true) {
    int k = 0;
    if (lane == 0) k = (int)atomicAdd(ticket, 1u);
    k = __shfl_sync(0xffffffffu, k, 0);
    if (k >= m) break;
    int r = r0 + k;
    int a = rp[k], e = rp[k + 1];
    T s = 0;
    for (int p = a + lane; p < e; p += 32) {
      int j = ldg_nc(ci + p);
      uint32_t spins = 0;
      while (ld_flag(flags + j) != epoch) {
        if (++spins > kWatchdogSpins) {
          if (st.error) *(volatile int*)st.error = 1;
          break;
        }
      }
      s += ldg_nc(val + p) * ld_strong(w + j);
    }
    s = warp_sum(s);
    if (lane == 0) {
      w[r] = (w[r] - s) / diag[r];
      st_flag_release(flags + r, epoch);
    }
  }
}

// Multi-RHS sync-free: a group of G lanes per component, lanes over RHS.
template <typename T, int G, int RPT>
__global__ void __launch_bounds__(256) tri_syncfree_multi(int r0, int m, const int* __restrict__ rp,
                                                          const int* __restrict__ ci, const T* __restrict__ val,
                                                          const T* __restrict__ diag, T* __restrict__ w,
                                                          int* __restrict__ flags, SolveState st, int slot,
                                                          int nrhs) {
  const int lane = threadIdx.x % G;
  const unsigned gmask = G == 32 ? 0xffffffffu : (((1u << G) - 1u) << ((threadIdx.x & 31) / G * G));
  const int epoch = (int)*((volatile uint32_t*)st.epoch);
  uint32_t* ticket = st.tickets + slot;
  while (true) {
    int k = 0;
    if (lane == 0) k = (int)atomicAdd(ticket, 1u);
    k = __shfl_sync(gmask, k, 0, G);
    if (k >= m) break;
    int r = r0 + k;
    int a = rp[k], e = rp[k + 1];
    for (int c0 = 0; c0 < nrhs; c0 += G * RPT) {
      T acc[RPT];
#pragma unroll
      for (int t = 0; t < RPT; ++t) acc[t] = 0;
      for (int p = a; p < e; ++p) {
        int j = ldg_nc(ci + p);
        if (c0 == 0) {
          uint32_t spins = 0;
          while (ld_flag(flags + j) != epoch) {
            if (++spins > kWatchdogSpins) {
              if (st.error) *(volatile int*)st.error = 1;
              break;
            }
          }
        }
        T v = ldg_nc(val + p);
        const T* xr = w + (int64_t)j * nrhs + c0 + lane;
#pragma unroll
        for (int t = 0; t < RPT; ++t)
          if (c0 + lane + G * t < nrhs) acc[t] += v * ld_strong(xr + G * t);
      }
      T d = diag[r];
      T* wr = w + (int64_t)r * nrhs + c0 + lane;
#pragma unroll
      for (int t = 0; t < RPT; ++t)
        if (c0 + lane + G * t < nrhs) wr[G * t] = (wr[G * t] - acc[t]) / d;
    }
    __syncwarp(gmask);
    if (lane == 0) st_flag_release(flags + r, epoch);
  }
}

}  // namespace k
}  // namespace sptrsv
