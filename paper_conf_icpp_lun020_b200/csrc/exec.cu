// Device side: plan upload, the Alg 7 segment loop (IMPROVED-RECURSIVE-BLOCK-
// ALGORITHM) and kernel dispatch.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>

#include "internal.h"
#include "kernels.cuh"

namespace sptrsv {

#define CUDA_TRY(x)                                                                  \
  do {                                                                               \
    cudaError_t e_ = (x);                                                            \
    if (e_ != cudaSuccess)                                                           \
      return Error{SPTRSV_ERROR_CUDA, std::string(#x) + ": " + cudaGetErrorString(e_)}; \
  } while (0)

namespace {

size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

template <typename F>
void dispatch_multi(int nrhs, F&& f) {
  if (nrhs <= 8)
    f(std::integral_constant<int, 8>(), std::integral_constant<int, 1>());
  else if (nrhs <= 32)
    f(std::integral_constant<int, 32>(), std::integral_constant<int, 1>());
  else if (nrhs <= 64)
    f(std::integral_constant<int, 32>(), std::integral_constant<int, 2>());
  else if (nrhs <= 128)
    f(std::integral_constant<int, 32>(), std::integral_constant<int, 4>());
  else if (nrhs <= 256)
    f(std::integral_constant<int, 32>(), std::integral_constant<int, 8>());
  else
    f(std::integral_constant<int, 32>(), std::integral_constant<int, 16>());
}

inline unsigned cdiv(int64_t a, int64_t b) { return (unsigned)((a + b - 1) / b); }

// long rows -> a warp per component (L247 "a thread or a 32-thread warp")
inline bool tri_use_warp(const Segment& S) { return S.info.nnz_per_row > 8; }

// Shared-memory geometry of the TMA-staged chain kernel (227 KB per CTA).
// Overridable for tuning with SPTRSV_CHAIN_GEOM="NST,RMAX,EMAX,XW,LMAX".
k::ChainGeom chain_geometry(const Plan& p) {
  int NST, RMAX, EMAX, XW, LMAX;
  if (p.vbytes == 8) {
    NST = 4; RMAX = 1024; EMAX = 2048; XW = 4096; LMAX = 256;
  } else {
    NST = 4; RMAX = 2048; EMAX = 4096; XW = 4096; LMAX = 256;
  }
  if (const char* e = std::getenv("SPTRSV_CHAIN_GEOM")) {
    int a, b, c, d, f;
    if (std::sscanf(e, "%d,%d,%d,%d,%d", &a, &b, &c, &d, &f) == 5 && a >= 2 && b >= 1 && c >= 1 && d >= 1 &&
        (d & (d - 1)) == 0 && f >= 1) {
      NST = a; RMAX = b; EMAX = c; XW = d; LMAX = f;
    }
  }
  return p.vbytes == 8 ? k::chain_geom<double>(NST, RMAX, EMAX, XW, LMAX)
                       : k::chain_geom<float>(NST, RMAX, EMAX, XW, LMAX);
}

k::ChainGeom frozen_geometry(const Plan& p) {
  const int* g = p.chain_geom;
  return p.vbytes == 8 ? k::chain_geom<double>(g[0], g[1], g[2], g[3], g[4])
                       : k::chain_geom<float>(g[0], g[1], g[2], g[3], g[4]);
}

// Cut a chain triangle into stages of whole levels (rows <= RMAX, entries <=
// EMAX, levels <= LMAX); a level that does not fit is split by rows.  Leaves
// chain_recs empty when one row has more than EMAX entries (the unstaged
// chain kernel runs instead).
void build_chain_stages(Segment& S, const k::ChainGeom& g) {
  S.chain_recs.clear();
  const auto& I = S.info;
  if (I.kind != 0 || I.impl != SPTRSV_IMPL_TRI_CHAIN) return;
  const int m = I.row1 - I.row0;
  for (int r = 0; r < m; ++r)
    if (S.rp[r + 1] - S.rp[r] > g.EMAX) return;
  std::vector<int32_t> st = {0};
  int cur_r = 0, cur_e = 0, cur_l = 0;
  auto close = [&](int at) {
    if (at > st.back()) st.push_back(at);
    cur_r = cur_e = cur_l = 0;
  };
  for (int l = 0; l < I.nlevels; ++l) {
    int la = S.level_ptr[l], lb = S.level_ptr[l + 1];
    int lr = lb - la, le = S.rp[lb] - S.rp[la];
    if (cur_r + lr <= g.RMAX && cur_e + le <= g.EMAX && cur_l + 1 <= g.LMAX) {
      cur_r += lr; cur_e += le; cur_l += 1;
      continue;
    }
    close(la);
    if (lr <= g.RMAX && le <= g.EMAX) {
      cur_r = lr; cur_e = le; cur_l = 1;
      continue;
    }
    for (int r = la; r < lb; ++r) {  // split a wide level by rows
      int re = S.rp[r + 1] - S.rp[r];
      if (cur_r + 1 > g.RMAX || cur_e + re > g.EMAX) close(r);
      cur_r += 1; cur_e += re; cur_l = 1;
    }
  }
  close(m);
  // records {sa, sb, e0, e1, l0, nl, 0, 0}, each followed by the record of
  // stage s + NST (the one the producer issues when stage s is done)
  const int ns = (int)st.size() - 1;
  S.chain_recs.assign((size_t)ns * 16, 0);
  int l = 0;
  for (int s = 0; s < ns; ++s) {
    int sa = st[s], sb = st[s + 1];
    while (S.level_ptr[l + 1] <= sa) ++l;  // level containing sa
    int l_last = l;
    while (S.level_ptr[l_last + 1] < sb) ++l_last;  // level containing sb-1
    int32_t* R = &S.chain_recs[(size_t)s * 16];
    R[0] = sa; R[1] = sb; R[2] = S.rp[sa]; R[3] = S.rp[sb]; R[4] = l; R[5] = l_last - l + 2;
  }
  for (int s = 0; s + g.NST < ns; ++s)
    std::memcpy(&S.chain_recs[(size_t)s * 16 + 8], &S.chain_recs[(size_t)(s + g.NST) * 16], 32);
}

// ELL-staged chain (see k::tri_chain_ell): eligible when every row has <= 4
// dependencies, all inside the x window of their level.  Geometry: RMAX rows
// per stage, as many stages as fit in 227 KB next to the window.
void build_chain_ell(Segment& S, size_t vb) {
  S.ell_K = 0;
  S.ell_recs.clear();
  S.ell_data.clear();
  const auto& I = S.info;
  if (I.kind != 0 || I.impl != SPTRSV_IMPL_TRI_CHAIN || I.nlevels < 2) return;
  if (const char* e = std::getenv("SPTRSV_ELL"))
    if (e[0] == '0') return;
  const int m = I.row1 - I.row0;
  int K = 0;
  for (int r = 0; r < m; ++r) K = std::max(K, S.rp[r + 1] - S.rp[r]);
  if (K < 1 || K > 4) return;
  int RMAX = 2048, XW = 4096, NSTMAX = 4;
  if (const char* e = std::getenv("SPTRSV_ELL_GEOM")) {
    int a, b, c;
    if (std::sscanf(e, "%d,%d,%d", &a, &b, &c) == 3 && a >= 1 && b >= 2 && (b & (b - 1)) == 0 && c >= 2) {
      RMAX = a; XW = b; NSTMAX = c;
    }
  }
  // every dependency of a row in level l must satisfy j >= end(l) - XW
  for (int l = 0; l < I.nlevels; ++l) {
    const int L1 = S.level_ptr[l + 1];
    for (int r = S.level_ptr[l]; r < L1; ++r)
      for (int q = S.rp[r]; q < S.rp[r + 1]; ++q)
        if (S.ci[q] - I.row0 < L1 - XW) return;
  }
  const uint32_t sb_bytes = vb == 8 ? k::ell_stage_bytes<double>(K, RMAX) : k::ell_stage_bytes<float>(K, RMAX);
  const uint32_t fixed = k::al16((XW + 2) * (uint32_t)vb) + 256;
  const int NST = std::min<int>(NSTMAX, (int)((232448 - fixed) / (sb_bytes + 16)));
  if (NST < 2) return;
  // stage boundaries: whole levels where possible (<= RMAX rows, <= 256 levels)
  std::vector<int32_t> st = {0};
  int cur_r = 0, cur_l = 0;
  for (int l = 0; l < I.nlevels; ++l) {
    const int la = S.level_ptr[l], lb = S.level_ptr[l + 1], lr = lb - la;
    if (cur_r + lr <= RMAX && cur_l + 1 <= 256) {
      cur_r += lr;
      cur_l += 1;
      continue;
    }
    if (la > st.back()) st.push_back(la);
    cur_r = cur_l = 0;
    if (lr <= RMAX) {
      cur_r = lr;
      cur_l = 1;
      continue;
    }
    for (int r = la + RMAX; r < lb; r += RMAX) st.push_back(r);  // split a wide level
    cur_r = lb - st.back();
    cur_l = 1;
  }
  if (m > st.back()) st.push_back(m);
  const int ns = (int)st.size() - 1;
  S.ell_recs.assign((size_t)ns * 16, 0);
  size_t off = 0;
  std::vector<size_t> offs(ns);
  for (int q = 0; q < ns; ++q) {
    const int n = st[q + 1] - st[q], npad = (n + 3) & ~3;
    offs[q] = off;
    off += k::al16(K * npad * 4) + k::al16(K * npad * (uint32_t)vb);
  }
  S.ell_data.assign(off, 0);
  int l = 0;
  for (int q = 0; q < ns; ++q) {
    const int sa = st[q], sb = st[q + 1], n = sb - sa, npad = (n + 3) & ~3;
    while (S.level_ptr[l + 1] <= sa) ++l;
    int l_last = l;
    while (S.level_ptr[l_last + 1] < sb) ++l_last;
    int32_t* R = &S.ell_recs[(size_t)q * 16];
    R[0] = sa; R[1] = sb; R[2] = l; R[3] = l_last - l + 2; R[4] = (int32_t)(offs[q] / 16); R[5] = npad;
    int32_t* slots = (int32_t*)&S.ell_data[offs[q]];
    char* vals = &S.ell_data[offs[q] + k::al16(K * npad * 4)];
    for (int kk = 0; kk < K; ++kk)
      for (int i = 0; i < npad; ++i) slots[kk * npad + i] = XW;  // the zero slot
    for (int i = 0; i < n; ++i) {
      const int r = sa + i;
      int kk = 0;
      for (int qq = S.rp[r]; qq < S.rp[r + 1]; ++qq, ++kk) {
        slots[kk * npad + i] = (S.ci[qq] - I.row0) & (XW - 1);
        std::memcpy(vals + ((size_t)kk * npad + i) * vb, &S.val[(size_t)qq * vb], vb);
      }
    }
  }
  for (int q = 0; q + NST < ns; ++q)
    std::memcpy(&S.ell_recs[(size_t)q * 16 + 8], &S.ell_recs[(size_t)(q + NST) * 16], 32);
  // consumer warps: cover the 90th-percentile level width with 2 rows/thread
  std::vector<int> widths(I.nlevels);
  for (int q = 0; q < I.nlevels; ++q) widths[q] = S.level_ptr[q + 1] - S.level_ptr[q];
  std::nth_element(widths.begin(), widths.begin() + (I.nlevels * 9) / 10, widths.end());
  int w90 = widths[(I.nlevels * 9) / 10];
  // measured on B200 (C2): per-level cost is issue-bound and grows ~13
  // cycles per extra warp, so 8..12 warps x 2 rows beat 31 warps x 1 row
  int warps = std::max(4, std::min(12, (w90 + 2 * 32 - 1) / (2 * 32)));
  if (const char* e = std::getenv("SPTRSV_ELL_WARPS")) warps = std::atoi(e);
  S.ell_warps = std::max(1, std::min(31, warps));
  S.ell_K = K;
  S.ell_NST = NST;
  S.ell_RMAX = RMAX;
  S.ell_XW = XW;
}

template <typename T, int K>
Error launch_chain_ell(Plan& p, Segment& S, const T* bw, T* xs, cudaStream_t s) {
  const int NST = S.ell_NST, RMAX = S.ell_RMAX, XW = S.ell_XW;
  const uint32_t smem = NST * k::ell_stage_bytes<T>(K, RMAX) + k::al16((XW + 2) * (uint32_t)sizeof(T)) + NST * 16;
  constexpr int RPT = 2;
  static uint32_t attr_bytes = 0;  // per template instance
  if (smem > attr_bytes) {
    CUDA_TRY(cudaFuncSetAttribute(k::tri_chain_ell<T, K, RPT>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  (int)smem));
    attr_bytes = smem;
  }
  // consumer warps: enough that NC * RPT covers a typical level, at most 31
  int nc_warps = S.ell_warps;
  const int nst = (int)(S.ell_recs.size() / 16);
  long long* tr = nullptr;
  if (p.trace) {
    if (S.h_trace.size() < (size_t)nst * 3) S.h_trace.assign((size_t)nst * 3, 0);
    if (!S.d_trace) CUDA_TRY(cudaMalloc(&S.d_trace, (size_t)nst * 3 * 8));
    tr = (long long*)S.d_trace;
  }
  k::tri_chain_ell<T, K, RPT><<<1, 32 * (nc_warps + 1), smem, s>>>(
      S.info.row0, nst, (const k::EllRec*)S.d_ell_recs, S.d_level_ptr, S.d_ell_data, bw, xs, NST, RMAX, XW, tr);
  return {SPTRSV_SUCCESS, ""};
}

template <typename T>
Error run_segments(Plan& p, T* bw, T* xs, int nrhs, cudaStream_t s, k::SolveState st, cudaEvent_t* ev) {
  for (size_t si = 0; si < p.segs.size(); ++si) {
    Segment& S = p.segs[si];
    const auto& I = S.info;
    const int m = I.row1 - I.row0;
    const T* val = (const T*)S.d_val;
    if (I.kind == 1) {  // square: b -= A x
      if (S.nzr > 0 && I.nnz > 0) {
        bool dcsr = I.format == SPTRSV_FMT_DCSR;
        if (nrhs == 1) {
          if (I.impl == SPTRSV_IMPL_SQ_VECTOR) {
            unsigned g = cdiv((int64_t)S.nzr * 32, 256);
            if (dcsr)
              k::sq_vector_1<T, true><<<g, 256, 0, s>>>(S.nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs, bw);
            else
              k::sq_vector_1<T, false><<<g, 256, 0, s>>>(S.nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs, bw);
          } else {
            unsigned g = cdiv(S.nzr, 256);
            if (dcsr)
              k::sq_scalar_1<T, true><<<g, 256, 0, s>>>(S.nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs, bw);
            else
              k::sq_scalar_1<T, false><<<g, 256, 0, s>>>(S.nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs, bw);
          }
        } else {
          dispatch_multi(nrhs, [&](auto G, auto R) {
            unsigned g = cdiv((int64_t)S.nzr * G, 256);
            if (dcsr)
              k::sq_multi<T, G, R, true><<<g, 256, 0, s>>>(S.nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs, bw,
                                                           nrhs);
            else
              k::sq_multi<T, G, R, false><<<g, 256, 0, s>>>(S.nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs, bw,
                                                            nrhs);
          });
        }
      }
    } else if (m > 0) {  // triangle: x_seg = L_seg^{-1} b_seg
      switch (I.impl) {
        case SPTRSV_IMPL_TRI_DIAG:
          k::tri_diag<T><<<cdiv((int64_t)m * nrhs, 256), 256, 0, s>>>(I.row0, m, nrhs, bw, xs);
          break;
        case SPTRSV_IMPL_TRI_LEVELSET: {
          const bool warp = tri_use_warp(S);
          for (int l = 0; l < I.nlevels; ++l) {
            int ra = I.row0 + S.level_ptr[l], rb = I.row0 + S.level_ptr[l + 1];
            if (rb <= ra) continue;
            if (nrhs == 1) {
              if (warp)
                k::tri_level_1<T, true><<<cdiv((int64_t)(rb - ra) * 32, 256), 256, 0, s>>>(
                    ra, rb, I.row0, S.d_rp, S.d_ci, val, bw, xs);
              else
                k::tri_level_1<T, false><<<cdiv(rb - ra, 256), 256, 0, s>>>(ra, rb, I.row0, S.d_rp, S.d_ci, val,
                                                                          bw, xs);
            } else {
              dispatch_multi(nrhs, [&](auto G, auto R) {
                k::tri_level_multi<T, G, R><<<cdiv((int64_t)(rb - ra) * G, 256), 256, 0, s>>>(
                    ra, rb, I.row0, S.d_rp, S.d_ci, val, bw, xs, nrhs);
              });
            }
          }
          break;
        }
        case SPTRSV_IMPL_TRI_CHAIN: {
          if (nrhs == 1 && S.ell_K > 0) {
            Error e;
            switch (S.ell_K) {
              case 1: e = launch_chain_ell<T, 1>(p, S, bw, xs, s); break;
              case 2: e = launch_chain_ell<T, 2>(p, S, bw, xs, s); break;
              case 3: e = launch_chain_ell<T, 3>(p, S, bw, xs, s); break;
              default: e = launch_chain_ell<T, 4>(p, S, bw, xs, s); break;
            }
            if (e.status) return e;
          } else if (nrhs == 1 && !S.chain_recs.empty()) {
            const k::ChainGeom cg = frozen_geometry(p);
            const uint32_t smem = k::chain_smem_bytes<T>(cg);
            static uint32_t attr_bytes = 0;  // per template instance
            if (smem > attr_bytes) {
              CUDA_TRY(cudaFuncSetAttribute(k::tri_chain_tma<T>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                            (int)smem));
              attr_bytes = smem;
            }
            const int nst = (int)(S.chain_recs.size() / 16);
            long long* tr = nullptr;
            if (p.trace) {  // debug: SPTRSV_TRACE=1, per-stage clock64 stamps
              if (S.h_trace.size() < (size_t)nst * 3) S.h_trace.assign((size_t)nst * 3, 0);
              if (!S.d_trace) CUDA_TRY(cudaMalloc(&S.d_trace, (size_t)nst * 3 * 8));
              tr = (long long*)S.d_trace;
            }
            k::tri_chain_tma<T><<<1, 1024, smem, s>>>(I.row0, nst, (const k::StageRec*)S.d_chain_recs,
                                                      S.d_level_ptr, S.d_rp, S.d_ci, val, bw, xs, cg, tr);
          } else if (nrhs == 1) {
            if (tri_use_warp(S))
              k::tri_chain_1<T, true><<<1, 1024, 0, s>>>(I.row0, I.nlevels, S.d_level_ptr, S.d_rp, S.d_ci, val,
                                                        bw, xs);
            else
              k::tri_chain_1<T, false><<<1, 1024, 0, s>>>(I.row0, I.nlevels, S.d_level_ptr, S.d_rp, S.d_ci, val,
                                                         bw, xs);
          } else {
            dispatch_multi(nrhs, [&](auto G, auto R) {
              k::tri_chain_multi<T, G, R><<<1, 1024, 0, s>>>(I.row0, I.nlevels, S.d_level_ptr, S.d_rp, S.d_ci,
                                                            val, bw, xs, nrhs);
            });
          }
          break;
        }
        default: {  // SPTRSV_IMPL_TRI_SYNCFREE
          const int cap = p.sm_count * 8;  // 8 CTAs x 8 warps per SM
          if (nrhs == 1) {
            if (tri_use_warp(S))
              k::tri_syncfree_warp<T, 4><<<std::min<unsigned>(cdiv(m, 8), cap), 256, 0, s>>>(
                  I.row0, m, S.d_rp, S.d_ci, val, bw, xs, st, S.ticket_slot);
            else
              k::tri_syncfree_thread<T, 4><<<std::min<unsigned>(cdiv(m, 256), cap), 256, 0, s>>>(
                  I.row0, m, S.d_rp, S.d_ci, val, bw, xs, st, S.ticket_slot);
          } else {
            dispatch_multi(nrhs, [&](auto G, auto R) {
              k::tri_syncfree_multi<T, G, R><<<std::min<unsigned>(cdiv((int64_t)m * G, 256), cap), 256, 0, s>>>(
                  I.row0, m, S.d_rp, S.d_ci, val, bw, xs, st, S.ticket_slot, nrhs);
            });
          }
          break;
        }
      }
    }
    if (ev) CUDA_TRY(cudaEventRecord(ev[2 + si], s));
  }
  return {SPTRSV_SUCCESS, ""};
}

int count_launches(const Plan& p) {
  int c = 2;  // permute in / out
  for (auto& S : p.segs) {
    if (S.info.kind == 1) {
      c += (S.nzr > 0 && S.info.nnz > 0);
    } else if (S.info.row1 > S.info.row0) {
      if (S.info.impl == SPTRSV_IMPL_TRI_LEVELSET) {
        for (int l = 0; l < S.info.nlevels; ++l) c += S.level_ptr[l + 1] > S.level_ptr[l];
      } else {
        c += 1;
      }
    }
  }
  return c;
}

// Debug (SPTRSV_TRACE=1): per-stage cycle breakdown of the staged chain
// kernel -- time spent waiting for the TMA stage vs walking its levels.
void dump_trace(Plan& p, cudaStream_t s) {
  cudaStreamSynchronize(s);
  for (size_t si = 0; si < p.segs.size(); ++si) {
    Segment& S = p.segs[si];
    if (!S.d_trace) continue;
    const int nst = S.ell_K ? (int)(S.ell_recs.size() / 16) : (int)(S.chain_recs.size() / 16);
    cudaMemcpy(S.h_trace.data(), S.d_trace, (size_t)nst * 24, cudaMemcpyDeviceToHost);
    long long wait = 0, work = 0, gap = 0;
    for (int k2 = 0; k2 < nst; ++k2) {
      wait += S.h_trace[3 * k2 + 1] - S.h_trace[3 * k2];
      work += S.h_trace[3 * k2 + 2] - S.h_trace[3 * k2 + 1];
      if (k2) gap += S.h_trace[3 * k2] - S.h_trace[3 * k2 - 1];
    }
    long long tot = S.h_trace[3 * nst - 1] - S.h_trace[0];
    std::fprintf(stderr,
                 "[sptrsv trace] seg %zu: %d stages, %d levels, %lld cycles: tma-wait %.1f%%, walk %.1f%%, "
                 "issue %.1f%%; per stage %.0f cycles, per level %.0f cycles\n",
                 si, nst, S.info.nlevels, tot, 100.0 * wait / tot, 100.0 * work / tot, 100.0 * gap / tot,
                 (double)tot / nst, (double)tot / S.info.nlevels);
  }
}

template <typename T>
Error solve_device(Plan& p, const T* b, int64_t ldb, T* x, int64_t ldx, int nrhs, sptrsv_layout_t layout,
                   cudaStream_t s) {
  const int n = p.n;
  size_t need = (size_t)n * nrhs * sizeof(T);
  if (need > p.ws.w_bytes) {
    if (p.ws.bw) cudaFree(p.ws.bw);
    if (p.ws.xs) cudaFree(p.ws.xs);
    p.ws.bw = p.ws.xs = nullptr;
    p.ws.w_bytes = 0;
    // +256 B: the staged chain kernel's 16-byte-aligned TMA windows may read
    // up to 15 bytes past the last row
    if (cudaMalloc(&p.ws.bw, need + 256) != cudaSuccess || cudaMalloc(&p.ws.xs, need + 256) != cudaSuccess) {
      cudaGetLastError();
      return {SPTRSV_ERROR_ALLOC, "workspace allocation failed"};
    }
    p.ws.w_bytes = need;
  }
  T* bw = (T*)p.ws.bw;
  T* xs = (T*)p.ws.xs;
  const T* rd = (const T*)p.d_rdiag;
  const int fill = p.needs_sentinel ? 1 : 0;
  k::SolveState st{p.d_tickets, p.nticket, p.d_error};
  cudaEvent_t* ev = nullptr;
  if (p.profiling) {
    size_t need_ev = p.segs.size() + 3;
    while (p.events.size() < need_ev) {
      cudaEvent_t e;
      CUDA_TRY(cudaEventCreate(&e));
      p.events.push_back((void*)e);
    }
    ev = (cudaEvent_t*)p.events.data();
    CUDA_TRY(cudaEventRecord(ev[0], s));
  }
  const int* iperm = p.d_perm + n;  // old -> new, stored right after perm
  if (nrhs == 1) {
    int64_t stride = layout == SPTRSV_ROW_MAJOR ? ldb : 1;
    k::perm_in_1<T><<<std::max(1u, cdiv(n, 256)), 256, 0, s>>>(n, p.d_perm, rd, b, stride, bw, xs, fill, st);
  } else if (layout == SPTRSV_COL_MAJOR) {
    dim3 g(std::max(1u, cdiv(n, 32)), cdiv(nrhs, 32));
    k::perm_in_cm<T><<<g, dim3(32, 8), 0, s>>>(n, nrhs, iperm, rd, b, ldb, bw, xs, fill, st);
  } else {
    k::perm_in_rm<T><<<std::max(1u, cdiv((int64_t)n * nrhs, 256)), 256, 0, s>>>(n, nrhs, p.d_perm, rd, b, ldb, bw,
                                                                                 xs, fill, st);
  }
  CUDA_TRY(cudaGetLastError());
  if (ev) CUDA_TRY(cudaEventRecord(ev[1], s));
  Error e = run_segments<T>(p, bw, xs, nrhs, s, st, ev);
  if (e.status) return e;
  CUDA_TRY(cudaGetLastError());
  if (nrhs == 1) {
    int64_t stride = layout == SPTRSV_ROW_MAJOR ? ldx : 1;
    k::perm_out_1<T><<<std::max(1u, cdiv(n, 256)), 256, 0, s>>>(n, p.d_perm, xs, x, stride);
  } else if (layout == SPTRSV_COL_MAJOR) {
    dim3 g(std::max(1u, cdiv(n, 32)), cdiv(nrhs, 32));
    k::perm_out_cm<T><<<g, dim3(32, 8), 0, s>>>(n, nrhs, iperm, xs, x, ldx);
  } else {
    k::perm_out_rm<T><<<std::max(1u, cdiv((int64_t)n * nrhs, 256)), 256, 0, s>>>(n, nrhs, p.d_perm, xs, x, ldx);
  }
  CUDA_TRY(cudaGetLastError());
  if (ev) {
    CUDA_TRY(cudaEventRecord(ev[2 + p.segs.size()], s));
    p.last_nseg_timed = (int)p.segs.size();
  }
  if (p.trace) dump_trace(p, s);
  return {SPTRSV_SUCCESS, ""};
}

bool is_device_ptr(const void* ptr) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, ptr) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

}  // namespace

Error upload(Plan& p, void* stream_v) {
  cudaStream_t s = (cudaStream_t)stream_v;
  const size_t vb = p.vbytes;
  const int n = p.n;
  // ---- arena layout (one allocation, segments in execution order, L229) ----
  size_t off = 0;
  auto take = [&](size_t bytes) {
    size_t o = off;
    off = align_up(off + bytes, 256);
    return o;
  };
  size_t o_perm = take((size_t)2 * n * 4);  // perm (new->old) then iperm (old->new)
  size_t o_rdiag = take((size_t)n * vb);
  struct Offs { size_t rp, ci, val, rows, lp, st, er, ed; };
  std::vector<Offs> so(p.segs.size());
  p.trace = std::getenv("SPTRSV_TRACE") != nullptr;
  const k::ChainGeom cg = chain_geometry(p);
  p.chain_geom[0] = cg.NST; p.chain_geom[1] = cg.RMAX; p.chain_geom[2] = cg.EMAX;
  p.chain_geom[3] = cg.XW; p.chain_geom[4] = cg.LMAX;
  p.nticket = 0;
  p.needs_sentinel = false;
  for (size_t i = 0; i < p.segs.size(); ++i) {
    Segment& S = p.segs[i];
    build_chain_stages(S, cg);
    build_chain_ell(S, vb);
    so[i].er = take(S.ell_recs.size() * 4);
    so[i].ed = take(S.ell_data.size());
    so[i].rp = take(S.rp.size() * 4);
    so[i].ci = take(S.ci.size() * 4);
    so[i].val = take(S.val.size());
    so[i].rows = take(S.rows.size() * 4);
    so[i].lp = take(S.level_ptr.size() * 4);
    so[i].st = take(S.chain_recs.size() * 4);
    if (S.info.kind == 0) S.ticket_slot = p.nticket++;
    if (S.info.kind == 0 && S.info.impl == SPTRSV_IMPL_TRI_SYNCFREE) p.needs_sentinel = true;
  }
  size_t o_tickets = take((size_t)std::max(1, p.nticket) * 4);
  p.arena_bytes = off;

  int dev;
  CUDA_TRY(cudaGetDevice(&dev));
  p.device = dev;
  if (cudaMalloc(&p.arena, std::max<size_t>(off, 256)) != cudaSuccess) {
    cudaGetLastError();
    return {SPTRSV_ERROR_ALLOC, "plan arena allocation failed (" + std::to_string(off) + " bytes)"};
  }
  // host staging of the whole arena, then one copy
  std::vector<char> h(off, 0);
  std::vector<int32_t> iperm(n);
  // p.perm is already in ORIGINAL indexing (UPPER: composed with J), so the
  // kernels gather b[perm[k]] / scatter x[perm[k]] directly.
  for (int k2 = 0; k2 < n; ++k2) iperm[p.perm[k2]] = k2;
  std::memcpy(&h[o_perm], p.perm.data(), (size_t)n * 4);
  std::memcpy(&h[o_perm + (size_t)n * 4], iperm.data(), (size_t)n * 4);
  std::memcpy(&h[o_rdiag], p.rdiag_new.data(), (size_t)n * vb);
  char* A = (char*)p.arena;
  for (size_t i = 0; i < p.segs.size(); ++i) {
    Segment& S = p.segs[i];
    std::memcpy(&h[so[i].rp], S.rp.data(), S.rp.size() * 4);
    std::memcpy(&h[so[i].ci], S.ci.data(), S.ci.size() * 4);
    std::memcpy(&h[so[i].val], S.val.data(), S.val.size());
    std::memcpy(&h[so[i].rows], S.rows.data(), S.rows.size() * 4);
    std::memcpy(&h[so[i].lp], S.level_ptr.data(), S.level_ptr.size() * 4);
    std::memcpy(&h[so[i].st], S.chain_recs.data(), S.chain_recs.size() * 4);
    S.d_rp = (const int32_t*)(A + so[i].rp);
    S.d_ci = (const int32_t*)(A + so[i].ci);
    S.d_val = (const void*)(A + so[i].val);
    S.d_rows = (const int32_t*)(A + so[i].rows);
    S.d_level_ptr = (const int32_t*)(A + so[i].lp);
    S.d_chain_recs = (const int32_t*)(A + so[i].st);
    std::memcpy(&h[so[i].er], S.ell_recs.data(), S.ell_recs.size() * 4);
    std::memcpy(&h[so[i].ed], S.ell_data.data(), S.ell_data.size());
    S.d_ell_recs = (const int32_t*)(A + so[i].er);
    S.d_ell_data = (const char*)(A + so[i].ed);
  }
  p.d_perm = (const int32_t*)(A + o_perm);
  p.d_rdiag = (const void*)(A + o_rdiag);
  p.d_tickets = (uint32_t*)(A + o_tickets);
  CUDA_TRY(cudaMemcpyAsync(p.arena, h.data(), off, cudaMemcpyHostToDevice, s));
  // mapped host word for the spin-wait watchdog
  if (cudaHostAlloc((void**)&p.h_error, sizeof(int32_t), cudaHostAllocMapped) == cudaSuccess) {
    *p.h_error = 0;
    CUDA_TRY(cudaHostGetDevicePointer((void**)&p.d_error, p.h_error, 0));
  } else {
    cudaGetLastError();
    p.h_error = nullptr;
    p.d_error = nullptr;
  }
  CUDA_TRY(cudaStreamSynchronize(s));
  p.launches_per_solve = count_launches(p);
  return {SPTRSV_SUCCESS, ""};
}

Error solve(Plan& p, const void* b, int64_t ldb, void* x, int64_t ldx, int32_t nrhs, sptrsv_layout_t layout,
            void* stream_v) {
  cudaStream_t s = (cudaStream_t)stream_v;
  if (p.h_error && *(volatile int32_t*)p.h_error) {
    *(volatile int32_t*)p.h_error = 0;
    return {SPTRSV_ERROR_DEADLOCK, "a spin-wait watchdog tripped during an earlier solve on this plan"};
  }
  if (nrhs == 0 || p.n == 0) return {SPTRSV_SUCCESS, ""};
  // the plan is bound to its device (our runtime's current device is not
  // torch's: make it explicit on every call)
  int cur = -1;
  if (cudaGetDevice(&cur) != cudaSuccess || cur != p.device) CUDA_TRY(cudaSetDevice(p.device));
  bool bd = is_device_ptr(b), xd = is_device_ptr(x);
  if (bd != xd) return {SPTRSV_ERROR_INVALID_VALUE, "b and x must both be device or both be host pointers"};
  const size_t vb = p.vbytes;
  if (bd) {
    if (p.dtype == SPTRSV_R64F)
      return solve_device<double>(p, (const double*)b, ldb, (double*)x, ldx, nrhs, layout, s);
    return solve_device<float>(p, (const float*)b, ldb, (float*)x, ldx, nrhs, layout, s);
  }
  // host buffers: stage through the device (end-to-end path), then sync
  size_t need = (size_t)p.n * nrhs * vb;
  if (need > p.ws.stage_bytes) {
    if (p.ws.stage_b) cudaFree(p.ws.stage_b);
    if (p.ws.stage_x) cudaFree(p.ws.stage_x);
    p.ws.stage_b = p.ws.stage_x = nullptr;
    p.ws.stage_bytes = 0;
    if (cudaMalloc(&p.ws.stage_b, need) != cudaSuccess || cudaMalloc(&p.ws.stage_x, need) != cudaSuccess) {
      cudaGetLastError();
      return {SPTRSV_ERROR_ALLOC, "staging allocation failed"};
    }
    p.ws.stage_bytes = need;
  }
  // compact copies: col-major n x nrhs (ld n) or row-major n x nrhs (ld nrhs)
  size_t width, height;
  int64_t dld;
  if (layout == SPTRSV_COL_MAJOR) {
    width = (size_t)p.n * vb;
    height = nrhs;
    dld = p.n;
  } else {
    width = (size_t)nrhs * vb;
    height = p.n;
    dld = nrhs;
  }
  CUDA_TRY(cudaMemcpy2DAsync(p.ws.stage_b, width, b, (size_t)ldb * vb, width, height, cudaMemcpyHostToDevice, s));
  Error e = p.dtype == SPTRSV_R64F
                ? solve_device<double>(p, (const double*)p.ws.stage_b, dld, (double*)p.ws.stage_x, dld, nrhs, layout, s)
                : solve_device<float>(p, (const float*)p.ws.stage_b, dld, (float*)p.ws.stage_x, dld, nrhs, layout, s);
  if (e.status) return e;
  CUDA_TRY(cudaMemcpy2DAsync(x, (size_t)ldx * vb, p.ws.stage_x, width, width, height, cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaStreamSynchronize(s));
  if (p.h_error && *(volatile int32_t*)p.h_error) {
    *(volatile int32_t*)p.h_error = 0;
    return {SPTRSV_ERROR_DEADLOCK, "spin-wait watchdog tripped"};
  }
  return {SPTRSV_SUCCESS, ""};
}

void release(Plan& p) {
  if (p.device >= 0) cudaDeviceSynchronize();
  if (p.arena) cudaFree(p.arena);
  if (p.ws.bw) cudaFree(p.ws.bw);
  if (p.ws.xs) cudaFree(p.ws.xs);
  if (p.ws.stage_b) cudaFree(p.ws.stage_b);
  if (p.ws.stage_x) cudaFree(p.ws.stage_x);
  if (p.h_error) cudaFreeHost(p.h_error);
  for (auto& S : p.segs)
    if (S.d_trace) cudaFree(S.d_trace);
  for (void* e : p.events) cudaEventDestroy((cudaEvent_t)e);
  p.arena = nullptr;
  p.ws = Workspace{};
  p.h_error = nullptr;
  p.events.clear();
}

// seg times helper used by the C ABI
Error seg_times(Plan& p, float* ms, int32_t cap, int32_t* count) {
  if (!p.profiling || p.events.size() < p.segs.size() + 3 || p.last_nseg_timed != (int)p.segs.size())
    return {SPTRSV_ERROR_INVALID_VALUE, "profiling is off or no solve was timed"};
  cudaEvent_t* ev = (cudaEvent_t*)p.events.data();
  int total = (int)p.segs.size() + 2;
  CUDA_TRY(cudaEventSynchronize(ev[p.segs.size() + 2]));
  for (int i = 0; i < total && i < cap; ++i) {
    float t = 0.f;
    CUDA_TRY(cudaEventElapsedTime(&t, ev[i], ev[i + 1]));
    ms[i] = t;
  }
  if (count) *count = total;
  return {SPTRSV_SUCCESS, ""};
}

Error device_info(int* sm_count, int* major, int* minor) {
  int dev;
  CUDA_TRY(cudaGetDevice(&dev));
  cudaDeviceProp pr;
  CUDA_TRY(cudaGetDeviceProperties(&pr, dev));
  *sm_count = pr.multiProcessorCount;
  *major = pr.major;
  *minor = pr.minor;
  return {SPTRSV_SUCCESS, ""};
}

}  // namespace sptrsv
