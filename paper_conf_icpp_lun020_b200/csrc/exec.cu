// Device side: plan upload, the Alg 7 segment loop (IMPROVED-RECURSIVE-BLOCK-
// ALGORITHM) and kernel dispatch.
#include <cuda_runtime.h>

#include <algorithm>
#include <numeric>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <mutex>
#include <unordered_map>
#include <array>

#include "internal.h"
#include "kernels.cuh"

namespace sptrsv {

#define CUDA_TRY(x)                                                                  \
  do {                                                                               \
    cudaError_t e_ = (x);                                                            \
    if (e_ != cudaSuccess)                                                           \
      return Error{SPTRSV_ERROR_CUDA, std::string(#x) + ": " + cudaGetErrorString(e_)}; \
  } while (0)

// Device memory of a plan: through the caller's hooks (the Python binding
// passes torch's caching allocator) or cudaMalloc / cudaFree.
void* dalloc(Plan& p, size_t bytes, cudaStream_t s) {
  if (p.opts.dev_alloc) return p.opts.dev_alloc(bytes, (void*)s, p.opts.alloc_ctx);
  void* q = nullptr;
  if (cudaMalloc(&q, bytes) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return q;
}
void dfree(Plan& p, void* q, cudaStream_t s) {
  if (!q) return;
  if (p.opts.dev_free)
    p.opts.dev_free(q, (void*)s, p.opts.alloc_ctx);
  else
    cudaFree(q);
}

namespace {

size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

// cudaFuncSetAttribute (max dynamic shared memory, non-portable cluster size)
// is per device: cache what was set per (kernel, device ordinal), under a
// mutex (plans may be solved from several threads and live on several GPUs).
std::mutex attr_mu;
std::unordered_map<std::string, uint32_t> attr_set;
cudaError_t ensure_smem_attr(const void* f, uint32_t smem, bool cluster) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  char key[64];  // the non-portable cluster attribute is part of the key
  std::snprintf(key, sizeof(key), "%p/%d/%d", f, dev, cluster ? 1 : 0);
  std::lock_guard<std::mutex> g(attr_mu);
  auto it = attr_set.find(key);
  if (it != attr_set.end() && it->second >= smem) return cudaSuccess;
  e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess && cluster) e = cudaFuncSetAttribute(f, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  if (e == cudaSuccess) attr_set[key] = smem;
  return e;
}

// Supernodal triangles with at least this many RHS run tri_supernode_multi
// (dense per-piece tiles over 64-column chunks); fewer columns would leave
// most of a chunk's lanes idle, so they take the sync-free SpTRSM kernel.
constexpr int kSnMultiMinRhs = 16;

// SpMM lane geometry for nrhs > 1: G lanes per row, RPT columns per lane per
// pass (capped by SPTRSV_SPMM="RPTMAX,UN" for tuning; default 8,2), UN row entries per
// gather round.  `multi_sync` is the sync-free triangle, which always uses
// UN = 1 (its polling is per entry).
SpmmCfg spmm_cfg() {
  SpmmCfg c;
  if (const char* e = std::getenv("SPTRSV_SPMM_TILE")) {  // RHS tile width of sq_multi_tiled (0 = off)
    const int t = std::atoi(e);
    c.tile = (t == 0 || t == 8 || t == 16 || t == 32) ? t : c.tile;
  }
  if (const char* e = std::getenv("SPTRSV_SPMM")) {
    int a, b;
    if (std::sscanf(e, "%d,%d", &a, &b) == 2 && (a == 1 || a == 2 || a == 4 || a == 8 || a == 16) && (b == 1 || b == 2)) {
      c.rpt_max = a;
      c.un = b;
    }
  }
  return c;
}

template <typename F>
void dispatch_rpt(int nrhs, int rpt_max, F&& f) {
  if (nrhs <= 8)
    f(std::integral_constant<int, 8>(), std::integral_constant<int, 1>());
  else if (nrhs <= 32 || rpt_max == 1)
    f(std::integral_constant<int, 32>(), std::integral_constant<int, 1>());
  else if (nrhs <= 64 || rpt_max == 2)
    f(std::integral_constant<int, 32>(), std::integral_constant<int, 2>());
  else if (nrhs <= 128 || rpt_max == 4)
    f(std::integral_constant<int, 32>(), std::integral_constant<int, 4>());
  else if (nrhs <= 256 || rpt_max == 8)
    f(std::integral_constant<int, 32>(), std::integral_constant<int, 8>());
  else
    f(std::integral_constant<int, 32>(), std::integral_constant<int, 16>());
}

template <typename F>
void dispatch_multi(int nrhs, F&& f) {
  dispatch_rpt(nrhs, 16, f);
}

template <typename F>
void dispatch_multi_un(int nrhs, const SpmmCfg& c, F&& f) {
  dispatch_rpt(nrhs, c.rpt_max, [&](auto G, auto R) {
    if (c.un == 2)
      f(G, R, std::integral_constant<int, 2>());
    else
      f(G, R, std::integral_constant<int, 1>());
  });
}

inline unsigned cdiv(int64_t a, int64_t b) { return (unsigned)((a + b - 1) / b); }

// long rows -> a warp per component (L247 "a thread or a 32-thread warp")
inline bool tri_use_warp(const Segment& S) {
  static const int thr = [] {
    const char* e = std::getenv("SPTRSV_SF_WARP_NPR");  // tuning: nnz/row above which a warp owns a row
    return e ? std::atoi(e) : 8;
  }();
  return S.info.nnz_per_row > thr;
}

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
// dependencies, all inside the x window of their level.  The triangle is cut
// into steps (levels; a level wider than NW*RG*32 rows is cut into chunks)
// of 32-row groups, steps into stages (<= RMAX rows, <= PMAX padded rows,
// <= SMAX steps, never wrapping the window) that fit NST buffers next to the
// window in 227 KB.
struct EllGeom {
  int XW, NST, RMAX, PMAX, SMAX;
};

EllGeom ell_geometry(int K, size_t vb) {
  EllGeom g{4096, 3, 1024, 1536, 128};
  if (const char* e = std::getenv("SPTRSV_ELL_GEOM")) {
    int a, b, c;
    if (std::sscanf(e, "%d,%d,%d", &a, &b, &c) == 3 && a >= 64 && b >= 2 && (b & (b - 1)) == 0 && c >= 2) {
      g.RMAX = a; g.XW = b; g.NST = c;
    }
  }
  // shrink the stage until NST buffers + window fit (and NST stages fit the window)
  for (;;) {
    g.PMAX = g.RMAX + g.RMAX / 2;
    const uint32_t sb = vb == 8 ? k::ell_stage_bytes<double>(K, g.RMAX, g.PMAX, g.SMAX)
                                : k::ell_stage_bytes<float>(K, g.RMAX, g.PMAX, g.SMAX);
    const size_t tot = (size_t)g.NST * sb + k::al16((g.XW + 2) * (uint32_t)vb) + 16 * g.NST;
    if ((tot <= 232448 && (size_t)(g.NST + 1) * g.RMAX <= (size_t)g.XW) || g.RMAX <= 128) break;
    g.RMAX -= 128;
  }
  return g;
}

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
  const EllGeom G = ell_geometry(K, vb);
  const int XW = G.XW;
  // every dependency of a row in level l must satisfy j >= end(l) - XW
  for (int l = 0; l < I.nlevels; ++l) {
    const int L1 = S.level_ptr[l + 1];
    for (int r = S.level_ptr[l]; r < L1; ++r)
      for (int q = S.rp[r]; q < S.rp[r + 1]; ++q)
        if (S.ci[q] - I.row0 < L1 - XW) return;
  }
  // consumer warps: cover the 90th-percentile level width with RG = 2 groups each
  std::vector<int> widths(I.nlevels);
  for (int q = 0; q < I.nlevels; ++q) widths[q] = S.level_ptr[q + 1] - S.level_ptr[q];
  std::nth_element(widths.begin(), widths.begin() + (I.nlevels * 9) / 10, widths.end());
  const int w90 = widths[(I.nlevels * 9) / 10];
  const int RG = 2;
  int warps = std::max(4, std::min(16, (w90 + RG * 32 - 1) / (RG * 32)));
  if (const char* e = std::getenv("SPTRSV_ELL_WARPS")) warps = std::atoi(e);
  warps = std::max(1, std::min(31, warps));
  const int cap = warps * RG * 32;  // rows per step
  // steps: {row_start, nrows} (triangle-local rows)
  // (a level is also cut where its rows cross a multiple of XW in global row
  // numbering, so no step wraps the window; running the two chunks of a
  // level one after the other is valid: rows of a level are independent)
  std::vector<std::pair<int, int>> steps;
  for (int l = 0; l < I.nlevels; ++l) {
    const int lb = S.level_ptr[l + 1];
    for (int a = S.level_ptr[l]; a < lb;) {
      const int to_wrap = XW - (int)(((uint32_t)(I.row0 + a)) & ((uint32_t)XW - 1));
      const int nr = std::min({cap, lb - a, to_wrap});
      steps.push_back({a, nr});
      a += nr;
    }
  }
  // stages
  struct St { int s0, s1, sa, sb, npad; };
  std::vector<St> stages;
  const uint32_t mask = (uint32_t)XW - 1;
  {
    St cur{0, 0, 0, 0, 0};
    for (int q = 0; q < (int)steps.size(); ++q) {
      const int ra = steps[q].first, nr = steps[q].second;
      const int padded = (nr + 31) / 32 * 32;
      // a stage never wraps the window: rows [sa, sb) must have contiguous slots
      const uint32_t slot0 = ((uint32_t)(I.row0 + cur.sa)) & mask;
      const bool fits = cur.s1 > cur.s0 && (ra + nr - cur.sa) <= G.RMAX && cur.npad + padded <= G.PMAX &&
                        cur.s1 - cur.s0 < G.SMAX && slot0 + (uint32_t)(ra + nr - cur.sa) <= (uint32_t)XW;
      if (cur.s1 > cur.s0 && !fits) {
        stages.push_back(cur);
        cur = St{q, q, ra, ra, 0};
      }
      if (cur.s1 == cur.s0) cur = St{q, q, ra, ra, 0};
      // a single step that wraps the window on its own: split it at the wrap
      cur.s1 = q + 1;
      cur.sb = ra + nr;
      cur.npad += padded;
    }
    if (cur.s1 > cur.s0) stages.push_back(cur);
  }
  // a step whose rows wrap the window inside one stage would break the bulk
  // store; steps are <= cap rows and stages start fresh at wraps, so check
  for (auto& st : stages) {
    const uint32_t slot0 = ((uint32_t)(I.row0 + st.sa)) & mask;
    if (slot0 + (uint32_t)(st.sb - st.sa) > (uint32_t)XW || st.sb - st.sa > G.RMAX || st.npad > G.PMAX ||
        st.s1 - st.s0 > G.SMAX)
      return;  // geometry cannot hold this triangle: fall back to the CSR chain
  }
  const int W = (K + 1) / 2;
  const int ns = (int)stages.size();
  S.ell_recs.assign((size_t)ns * 16, 0);
  std::vector<size_t> offs(ns);
  size_t off = 0;
  for (int q = 0; q < ns; ++q) {
    const int npad = stages[q].npad;
    const size_t bytes = 16 * (size_t)(stages[q].s1 - stages[q].s0) + k::al16(W * npad * 4) + k::al16(K * npad * (uint32_t)vb);
    offs[q] = off;
    off += k::al16((uint32_t)bytes);
  }
  S.ell_data.assign(off, 0);
  for (int q = 0; q < ns; ++q) {
    const St& st = stages[q];
    const int nst = st.s1 - st.s0, npad = st.npad;
    char* blk = &S.ell_data[offs[q]];
    int32_t* srec = (int32_t*)blk;
    uint32_t* words = (uint32_t*)(blk + 16 * nst);
    char* vals = blk + 16 * nst + k::al16(W * npad * 4);
    const uint32_t zero = (uint32_t)XW;
    for (int w = 0; w < W; ++w)
      for (int i = 0; i < npad; ++i) words[w * npad + i] = zero | (zero << 16);
    int grp = 0;
    for (int t = st.s0; t < st.s1; ++t) {
      const int ra = steps[t].first, nr = steps[t].second, ng = (nr + 31) / 32;
      int32_t* R4 = srec + 4 * (t - st.s0);
      R4[0] = grp; R4[1] = ng; R4[2] = ra - st.sa; R4[3] = nr;
      for (int i = 0; i < nr; ++i) {
        const int r = ra + i, pi = grp * 32 + i;
        int kk = 0;
        for (int qq = S.rp[r]; qq < S.rp[r + 1]; ++qq, ++kk) {
          const uint32_t sl = ((uint32_t)S.ci[qq]) & mask;  // global permuted row -> window slot
          uint32_t& wd = words[(kk >> 1) * npad + pi];
          wd = (kk & 1) ? ((wd & 0xffffu) | (sl << 16)) : ((wd & 0xffff0000u) | sl);
          std::memcpy(vals + ((size_t)kk * npad + pi) * vb, &S.val[(size_t)qq * vb], vb);
        }
      }
      grp += ng;
    }
    int32_t* R = &S.ell_recs[(size_t)q * 16];
    const size_t bytes = 16 * (size_t)nst + k::al16(W * npad * 4) + k::al16(K * npad * (uint32_t)vb);
    R[0] = st.sa; R[1] = st.sb; R[2] = nst; R[3] = (int32_t)(offs[q] / 16); R[4] = (int32_t)k::al16((uint32_t)bytes);
    R[5] = npad;
  }
  for (int q = 0; q + G.NST < ns; ++q)
    std::memcpy(&S.ell_recs[(size_t)q * 16 + 8], &S.ell_recs[(size_t)(q + G.NST) * 16], 32);
  S.ell_warps = warps;
  S.ell_K = K;
  S.ell_NST = G.NST;
  S.ell_RMAX = G.RMAX;
  S.ell_PMAX = G.PMAX;
  S.ell_SMAX = G.SMAX;
  S.ell_XW = XW;
}

template <typename T, int K>
Error launch_chain_ell(Plan& p, Segment& S, const T* bw, T* xs, cudaStream_t s) {
  const int NST = S.ell_NST, RMAX = S.ell_RMAX, PMAX = S.ell_PMAX, SMAX = S.ell_SMAX, XW = S.ell_XW;
  const uint32_t smem = NST * k::ell_stage_bytes<T>(K, RMAX, PMAX, SMAX) + k::al16((XW + 2) * (uint32_t)sizeof(T)) +
                        NST * 16;
  constexpr int RG = 2;
  CUDA_TRY(ensure_smem_attr((const void*)k::tri_chain_ell<T, K, RG>, smem, false));
  const int nst = (int)(S.ell_recs.size() / 16);
  long long* tr = nullptr;
  if (p.trace) {
    if (S.h_trace.size() < (size_t)nst * 3) S.h_trace.assign((size_t)nst * 3, 0);
    if (!S.d_trace) CUDA_TRY(cudaMalloc(&S.d_trace, (size_t)nst * 3 * 8));
    tr = (long long*)S.d_trace;
  }
  k::tri_chain_ell<T, K, RG><<<1, 32 * (S.ell_warps + 1), smem, s>>>(
      S.info.row0, nst, (const k::EllRec*)S.d_ell_recs, S.d_ell_data, bw, xs, NST, RMAX, PMAX, SMAX, XW, tr);
  return {SPTRSV_SUCCESS, ""};
}

// Supernodal pieces (see k::tri_supernode): per piece its shared external
// column list, the dense external values V_J (column-major, ld = width) and
// the packed strictly-lower diagonal block.  Values are the D^-1-scaled ones
// of the segment (R27).
void build_supernodes(Segment& S, size_t vb, int32_t& part_base) {
  S.sn_desc.clear();
  S.sn_cols.clear();
  S.sn_vals.clear();
  S.sn_blk.clear();
  S.sn_items.clear();
  const auto& I = S.info;
  if (I.kind != 0 || I.impl != SPTRSV_IMPL_TRI_SUPERNODE) return;
  const int np = (int)S.sn_ptr.size() - 1;
  std::vector<k::SnDesc> desc(np);
  size_t nv = 0, nb = 0, nc = 0;
  for (int J = 0; J < np; ++J) {
    const int a = S.sn_ptr[J], w = S.sn_ptr[J + 1] - a;
    const int ne = S.rp[a + 1] - S.rp[a];
    desc[J] = k::SnDesc{I.row0 + a, w, ne, (int)nc, (long long)nv, (long long)nb};
    nc += ne;
    nv += (size_t)ne * w;
    nb += (size_t)w * (w - 1) / 2;
  }
  S.sn_cols.resize(nc);
  S.sn_vals.resize(std::max<size_t>(nv, 1) * vb);  // every byte is written below
  S.sn_blk.resize(std::max<size_t>(nb, 1) * vb);
  par_for(np, 0, [&](int64_t J0, int64_t J1) {
    for (int64_t J = J0; J < J1; ++J) {
      const k::SnDesc& d = desc[J];
      const int a = S.sn_ptr[J];
      std::memcpy(&S.sn_cols[d.coff], &S.ci[S.rp[a]], (size_t)d.ne * 4);
      for (int t = 0; t < d.w; ++t) {
        const int base = S.rp[a + t];
        for (int q = 0; q < d.ne; ++q)
          std::memcpy(&S.sn_vals[((size_t)d.voff + (size_t)q * d.w + t) * vb], &S.val[(size_t)(base + q) * vb], vb);
        for (int c = 0; c < t; ++c) {
          const size_t off = (size_t)d.boff + (size_t)c * (d.w - 1) - (size_t)c * (c - 1) / 2 + (t - c - 1);
          std::memcpy(&S.sn_blk[off * vb], &S.val[(size_t)(base + d.ne + c) * vb], vb);
        }
      }
    }
  }, 512);
  S.sn_desc.resize((size_t)np * sizeof(k::SnDesc));
  std::memcpy(S.sn_desc.data(), desc.data(), S.sn_desc.size());
  // work items (k::tri_supernode): long external lists cut into kSnChunk-
  // column chunks with 32-wide partial slots (SPTRSV_SN_NOSPLIT: whole pieces)
  const bool split = std::getenv("SPTRSV_SN_NOSPLIT") == nullptr;
  S.sn_part_base = (part_base + 31) / 32 * 32;
  int32_t nslot = 0;
  for (int J = 0; J < np; ++J) {
    const int ne = desc[J].ne;
    if (!split || ne <= k::kSnChunk) {
      const int32_t rec[8] = {J, 0, ne, 0, 0, 0, 0, 0};
      S.sn_items.insert(S.sn_items.end(), rec, rec + 8);
      continue;
    }
    const int first = nslot;
    for (int q0 = 0; q0 < ne; q0 += k::kSnChunk) {
      const int q1 = std::min(ne, q0 + k::kSnChunk);
      const bool last = q1 == ne;
      const int32_t rec[8] = {J, q0, q1, last ? 2 : 1, last ? first : nslot, last ? nslot : 0, 0, 0};
      if (!last) ++nslot;
      S.sn_items.insert(S.sn_items.end(), rec, rec + 8);
    }
  }
  part_base = S.sn_part_base + 32 * nslot;
}

// Strand wavefront (k::tri_wave): strands = contiguous ranges of the
// ORIGINAL (lower) row index balanced in rows, C CTAs (one cluster) x W warps;
// groups = <= 32 rows of one level of a strand; the device row order of the
// triangle becomes strand-major, group-major (wave_tau).  Leaves wave_K == 0
// and switches the segment to the chain kernel when the triangle does not
// suit it (a row with > 8 dependencies, or > 10% of the dependencies would
// have to be polled in global memory).
void build_wave(const Plan& p, Segment& S, size_t vb) {
  S.wave_K = 0;
  S.wave_tau.clear();
  S.wave_strands.clear();
  S.wave_data.clear();
  S.wave_crows.clear();
  auto& I = S.info;
  if (I.kind != 0 || I.impl != SPTRSV_IMPL_TRI_PIPE) return;
  const int m = I.row1 - I.row0;
  PhaseClock wclk;
  int C = 16, W = 2, GPC = k::kWaveGpcBig, NCH = 4;
  if (const char* e = std::getenv("SPTRSV_WAVE")) {
    int a, b2, c, d;
    if (std::sscanf(e, "%d,%d,%d,%d", &a, &b2, &c, &d) == 4 && a >= 1 && a <= 16 && b2 >= 1 && b2 <= 8 &&
        c >= 1 && c <= 32 && d >= 2 && d <= 4) {
      C = a; W = b2; GPC = c <= 6 ? 6 : k::kWaveGpcBig; NCH = d;
    }
  }
  auto give_up = [&]() {
    S.wave_K = 0;
    S.wave_tau.clear();
    I.impl = SPTRSV_IMPL_TRI_CHAIN;
  };
  int K = 0;
  for (int r = 0; r < m; ++r) K = std::max(K, S.rp[r + 1] - S.rp[r]);
  if (m < 1 || K < 1 || K > 8) return give_up();
  const int Kt = K <= 2 ? 2 : K <= 4 ? 4 : 8;
  // strands: contiguous runs of the original row index, cut so that no
  // strand holds more than `cap` rows of one level (cap = 32: one group per
  // level and strand).  A strand then needs one level step per level it
  // spans, and a strand that starts late (its rows sit in late levels) is
  // short: the critical path is ~ the number of levels, not the widest
  // strand's row count (equal-row strands made the last strands of C2's
  // anti-diagonal triangles 3-6 groups per level).  cap grows by 32 until
  // the strands fit the cluster (C_max x W warps).
  std::vector<int32_t> order(m), strand(m);
  {  // rows in ascending original index: the keys are distinct, so a slot
     // table over their range replaces a comparison sort (O(m + range))
    int32_t kmin = INT32_MAX, kmax = -1;
    for (int r = 0; r < m; ++r) {
      kmin = std::min(kmin, p.lower_old[I.row0 + r]);
      kmax = std::max(kmax, p.lower_old[I.row0 + r]);
    }
    std::vector<int32_t> slot((size_t)std::max(0, kmax - kmin + 1), -1);
    for (int r = 0; r < m; ++r) slot[p.lower_old[I.row0 + r] - kmin] = r;
    int q = 0;
    for (int32_t t : slot)
      if (t >= 0) order[q++] = t;
  }
  const int C_max = C;
  int NS = 0;
  {
    std::vector<int32_t> lvcnt(std::max(1, I.nlevels) + 1, 0), touched;
    for (int cap = 32;; cap += 32) {
      NS = 0;
      int cur = 0;
      for (int q = 0; q < m; ++q) {
        const int r = order[q];
        const int lv = p.leaf_level[I.row0 + r];
        if (q == 0 || lvcnt[lv] + 1 > cap) {  // open a new strand
          for (int t : touched) lvcnt[t] = 0;
          touched.clear();
          cur = NS++;
        }
        if (lvcnt[lv]++ == 0) touched.push_back(lv);
        strand[r] = cur;
      }
      for (int t : touched) lvcnt[t] = 0;
      touched.clear();
      if (NS <= C_max * W) break;
    }
  }
  C = std::max(1, (NS + W - 1) / W);
  if (const char* e = std::getenv("SPTRSV_WAVE_EQUAL")) {  // tuning: the old equal-row strands
    NS = C_max * W;
    C = C_max;
    for (int q = 0; q < m; ++q) strand[order[q]] = (int)((int64_t)q * NS / m);
  }
  NS = C * W;  // trailing strands of the last CTA stay empty
  // rows of every strand in level order (= local row order); groups
  std::vector<std::vector<int32_t>> srows(NS);
  for (int r = 0; r < m; ++r) srows[strand[r]].push_back(r);
  std::vector<int32_t> pos(m), qpos(m), s_start(NS + 1, 0);
  std::vector<std::vector<std::pair<int32_t, int32_t>>> groups(NS);  // (first pos, count) per strand
  int q = 0;
  for (int s2 = 0; s2 < NS; ++s2) {
    s_start[s2] = q;
    const auto& R = srows[s2];
    for (size_t a = 0; a < R.size();) {
      const int lv = p.leaf_level[I.row0 + R[a]];
      size_t b2 = a;
      while (b2 < R.size() && b2 - a < 32 && p.leaf_level[I.row0 + R[b2]] == lv) ++b2;
      groups[s2].push_back({(int32_t)a, (int32_t)(b2 - a)});
      a = b2;
    }
    for (size_t a = 0; a < R.size(); ++a) {
      pos[R[a]] = (int32_t)a;
      qpos[R[a]] = q++;
    }
  }
  s_start[NS] = q;
  wclk.lap("  wave: strands + groups");
  // own window: the smallest power of two covering every same-strand distance
  int maxd = 0;
  for (int r = 0; r < m; ++r)
    for (int e = S.rp[r]; e < S.rp[r + 1]; ++e) {
      const int j = S.ci[e] - I.row0;
      if (strand[j] == strand[r]) maxd = std::max(maxd, pos[r] - pos[j]);
    }
  int xw_cap = 4096;  // SPTRSV_WAVE_XW / SPTRSV_WAVE_ICAP: test hooks forcing the global-memory fallback
  if (const char* e = std::getenv("SPTRSV_WAVE_XW")) xw_cap = std::max(64, std::min(4096, std::atoi(e)));
  int XW = 64;
  while (XW < maxd + 32 && XW < xw_cap) XW *= 2;
  // shared-memory budget (E = 2 is the upper bound of the chunk size): the
  // deepest ring (GPC x NCH) that leaves >= 1024 import slots per strand
  const uint32_t gb2 = vb == 8 ? k::wave_group_bytes<double>(Kt, 2) : k::wave_group_bytes<float>(Kt, 2);
  uint32_t bring = 0;
  int64_t icap = -1;
  for (;;) {
    bring = vb == 8 ? k::wave_bring_bytes<double>(GPC) : k::wave_bring_bytes<float>(GPC);
    const int64_t rings = (int64_t)W * NCH * (k::wave_hdr_bytes(GPC) + (int64_t)GPC * gb2 + bring + 16);
    const int64_t slots_avail = (232448 - 512 - rings) / (int64_t)vb;
    icap = (slots_avail - 2) / W - XW;
    if (icap >= 1024 || (GPC == 6 && NCH == 2)) break;
    if (NCH > 2) --NCH;
    else { GPC = 6; NCH = 4; }
  }
  if (const char* e = std::getenv("SPTRSV_WAVE_ICAP")) icap = std::min<int64_t>(icap, std::max(0, std::atoi(e)));
  if (icap < 0) return give_up();
  // classify every dependency (rows in execution order so imports are
  // numbered in first-use order): kind 0 own, 1 import (strand, idx), 2 global
  struct Dep { int8_t kind; int32_t a, b; };
  std::vector<Dep> dep(S.ci.size());
  std::vector<int32_t> nimp(NS, 0);
  std::vector<uint8_t> npush(m, 0);
  std::vector<std::array<int32_t, 4>> push(m, {-1, -1, -1, -1});  // (strand, idx) x 2
  std::unordered_map<int64_t, int32_t> imp;
  int64_t nglobal = 0;
  for (int s2 = 0; s2 < NS; ++s2)
    for (int r : srows[s2])
      for (int e = S.rp[r]; e < S.rp[r + 1]; ++e) {
        const int j = S.ci[e] - I.row0;
        if (strand[j] == s2 && pos[r] - pos[j] <= XW - 32) {
          dep[e] = {0, j, 0};
          continue;
        }
        if (strand[j] != s2) {
          const int64_t key = (int64_t)s2 * m + j;
          auto it = imp.find(key);
          if (it != imp.end()) {
            dep[e] = {1, s2, it->second};
            continue;
          }
          if (npush[j] < 2 && nimp[s2] < icap) {
            const int idx = nimp[s2]++;
            imp.emplace(key, idx);
            push[j][2 * npush[j]] = s2;
            push[j][2 * npush[j] + 1] = idx;
            ++npush[j];
            dep[e] = {1, s2, idx};
            continue;
          }
        }
        dep[e] = {2, j, 0};
        ++nglobal;
      }
  wclk.lap("  wave: dependency classes");
  if (nglobal * 10 > (int64_t)S.ci.size() && p.opts.force_tri_impl != SPTRSV_IMPL_TRI_PIPE) return give_up();
  int E = 0;
  for (int r = 0; r < m; ++r) E = std::max<int>(E, npush[r]);
  // x-area layout per CTA: slots 0-1 zero, then per warp own window + imports
  std::vector<int32_t> own_base(NS), imp_base(NS);
  int xa = 2;
  for (int c = 0; c < C; ++c) {
    int cur = 2;
    for (int w = 0; w < W; ++w) {
      const int s2 = c * W + w;
      own_base[s2] = cur;
      cur += XW;
      imp_base[s2] = cur;
      cur += nimp[s2];
    }
    xa = std::max(xa, cur);
  }
  const uint32_t gbytes = vb == 8 ? k::wave_group_bytes<double>(Kt, E) : k::wave_group_bytes<float>(Kt, E);
  const uint32_t hbytes = k::wave_hdr_bytes(GPC);
  // first-use import list per chunk (what chunk_wait polls): its length
  std::vector<std::vector<std::vector<uint32_t>>> clist(NS);
  int max_ci = 0;
  {
    const uint32_t VB0 = (uint32_t)vb;
    for (int s2 = 0; s2 < NS; ++s2) {
      std::vector<char> seen(nimp[s2], 0);
      const auto& Gs = groups[s2];
      const auto& R = srows[s2];
      const int nch = (int)((Gs.size() + GPC - 1) / GPC);
      // one list per quarter (k::kWaveQ parts) of the chunk's groups
      clist[s2].resize((size_t)nch * k::kWaveQ);
      for (int c = 0; c < nch; ++c)
        for (int q = 0; q < k::kWaveQ; ++q) {
          auto& L = clist[s2][(size_t)c * k::kWaveQ + q];
          const int ga = c * GPC + q * GPC / k::kWaveQ, gb = c * GPC + (q + 1) * GPC / k::kWaveQ;
          for (int g2 = ga; g2 < std::min<int>((int)Gs.size(), gb); ++g2)
            for (int l = 0; l < Gs[g2].second; ++l) {
              const int r = R[Gs[g2].first + l];
              for (int e = S.rp[r]; e < S.rp[r + 1]; ++e)
                if (dep[e].kind == 1 && !seen[dep[e].b]) {
                  seen[dep[e].b] = 1;
                  L.push_back((uint32_t)(imp_base[s2] + dep[e].b) * VB0);
                }
            }
          max_ci = std::max<int>(max_ci, (int)L.size());
        }
    }
  }
  const int ipl = (max_ci + 31) / 32;
  const uint32_t cbytes = hbytes + (uint32_t)GPC * gbytes + (uint32_t)(ipl * k::kWaveQ) * 128u;
  {  // the import lists must still fit next to the x area (else: the chain kernel)
    const int64_t need = (int64_t)k::al16((uint32_t)xa * (uint32_t)vb) + (int64_t)W * NCH * (cbytes + bring + 16);
    if (need > 232448) return give_up();
  }
  // chunks
  std::vector<k::WaveStrand> sr(NS);
  std::vector<int32_t> nchunk(NS);
  size_t total = 0;
  for (int s2 = 0; s2 < NS; ++s2) {
    nchunk[s2] = (int)((groups[s2].size() + GPC - 1) / GPC);
    total += (size_t)nchunk[s2] * cbytes;
  }
  S.wave_data.assign(std::max<size_t>(total, 16), 0);
  size_t off = 0;
  const int r0 = I.row0;
  const uint32_t VB = (uint32_t)vb;
  auto word = [&](int e) -> uint32_t {  // byte offset in the x area, or bit 31 | global row
    const Dep& d = dep[e];
    if (d.kind == 0) return (uint32_t)(own_base[strand[d.a]] + (pos[d.a] & (XW - 1))) * VB;
    if (d.kind == 1) return (uint32_t)(imp_base[d.a] + d.b) * VB;
    return 0x80000000u | (uint32_t)(r0 + qpos[d.a]);
  };
  const int bshift_mask = vb == 8 ? 1 : 3;  // bw is 256-byte aligned: TMA window shift of row lo
  for (int s2 = 0; s2 < NS; ++s2) {
    k::WaveStrand& W2 = sr[s2];
    std::memset(&W2, 0, sizeof(W2));
    W2.off16 = (int)(off / 16);
    W2.nchunk = nchunk[s2];
    W2.ngroups = (int)groups[s2].size();
    W2.row0 = r0 + s_start[s2];
    W2.imp_lo = (uint32_t)imp_base[s2] * VB;
    W2.imp_hi = (uint32_t)(imp_base[s2] + nimp[s2]) * VB;
    const auto& Gs = groups[s2];
    const auto& R = srows[s2];
    auto chunk_rows = [&](int c, int& lo, int& hi) {
      const int g0 = c * GPC, g1 = std::min<int>((int)Gs.size(), g0 + GPC) - 1;
      lo = r0 + s_start[s2] + Gs[g0].first;
      hi = r0 + s_start[s2] + Gs[g1].first + Gs[g1].second;
    };
    for (int c = 0; c < nchunk[s2]; ++c) {
      char* B = &S.wave_data[off + (size_t)c * cbytes];
      int32_t* hdr = (int32_t*)B;
      chunk_rows(c, hdr[0], hdr[1]);
      if (c + NCH < nchunk[s2]) chunk_rows(c + NCH, hdr[2], hdr[3]);
      if (c < 4) chunk_rows(c, W2.lo[c], W2.hi[c]);
      const int lo = hdr[0];
      for (int gi = 0; gi < GPC; ++gi) {
        const int g = c * GPC + gi;
        int32_t* gh = (int32_t*)(B + 16) + 4 * gi;
        uint32_t* wd = (uint32_t*)(B + hbytes + (size_t)gi * gbytes);
        uint32_t* so = wd + 32 * Kt;
        uint32_t* pw = so + 32;
        char* vv = (char*)(pw + 32 * E);
        for (int l = 0; l < 32; ++l) so[l] = VB;  // sink slot (padding lanes)
        for (int l = 0; l < 32 * E; ++l) pw[l] = 0xffffffffu;
        if (g >= (int)Gs.size()) continue;  // padding group: never executed
        int flags = 0;
        gh[0] = r0 + s_start[s2] + Gs[g].first;
        gh[2] = gh[0] - lo + (lo & bshift_mask);
        for (int l = 0; l < Gs[g].second; ++l) {
          const int r = R[Gs[g].first + l];
          so[l] = (uint32_t)(own_base[s2] + (pos[r] & (XW - 1))) * VB;
          int kk = 0;
          for (int e = S.rp[r]; e < S.rp[r + 1]; ++e, ++kk) {
            wd[kk * 32 + l] = word(e);
            if (dep[e].kind == 2) flags |= k::kWaveGF_GLOBAL;
            std::memcpy(vv + ((size_t)kk * 32 + l) * vb, &S.val[(size_t)e * vb], vb);
          }
          for (int e2 = 0; e2 < npush[r]; ++e2) {
            const int cs = push[r][2 * e2], ci2 = push[r][2 * e2 + 1];
            pw[e2 * 32 + l] = ((uint32_t)(cs / W) << 24) | ((uint32_t)(imp_base[cs] + ci2) * VB);
            flags |= k::kWaveGF_PUSH;
          }
        }
        gh[1] = Gs[g].second | flags;
      }
      for (int q = 0; q < k::kWaveQ; ++q) {  // rest of each list: 0 = the zero slot
        uint32_t* il = (uint32_t*)(B + hbytes + (size_t)GPC * gbytes + (size_t)q * ipl * 128);
        const auto& L = clist[s2][(size_t)c * k::kWaveQ + q];
        for (size_t i = 0; i < L.size(); ++i) il[i] = L[i];
      }
    }
    off += (size_t)nchunk[s2] * cbytes;
  }
  wclk.lap("  wave: chunks");
  S.wave_strands.resize(sizeof(k::WaveStrand) * NS);
  std::memcpy(S.wave_strands.data(), sr.data(), S.wave_strands.size());
  S.wave_tau.assign(m, 0);
  for (int r = 0; r < m; ++r) S.wave_tau[qpos[r]] = r;
  S.wave_K = Kt;
  S.wave_E = E;
  S.wave_C = C;
  S.wave_W = W;
  S.wave_GPC = GPC;
  S.wave_NCH = NCH;
  S.wave_XW = XW;
  S.wave_xa = xa;
  S.wave_chunk_bytes = cbytes;
  S.wave_bring_bytes = bring;
  S.wave_group_bytes = gbytes;
  S.wave_ipl = ipl;
  S.wave_global = nglobal;
}

template <typename T, int K, int E, int GPC, bool GLB>
Error launch_wave_t(Plan& p, Segment& S, const T* bw, T* xs, k::SolveState st, cudaStream_t s) {
  k::WaveGeom g{S.wave_W,           S.wave_GPC,         S.wave_NCH,         S.wave_xa,
                S.wave_chunk_bytes, S.wave_bring_bytes, S.wave_group_bytes, k::wave_hdr_bytes(S.wave_GPC),
                S.wave_ipl};
  const uint32_t smem = k::wave_smem_bytes<T>(g);
  auto kern = k::tri_wave<T, K, E, GPC, GLB>;
  CUDA_TRY(ensure_smem_attr((const void*)kern, smem, true));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(S.wave_C);
  cfg.blockDim = dim3(32 * (S.wave_W + 1));  // + the TMA producer warp
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = S.wave_C;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  long long* tr = nullptr;
  if (p.trace) {  // debug: SPTRSV_TRACE=1, per-strand clock64 stamps
    const size_t nt = (size_t)S.wave_C * S.wave_W * 1024;
    if (S.h_trace.size() < nt) S.h_trace.assign(nt, 0);
    if (!S.d_trace) CUDA_TRY(cudaMalloc(&S.d_trace, nt * 8));
    CUDA_TRY(cudaMemsetAsync(S.d_trace, 0, nt * 8, s));
    tr = (long long*)S.d_trace;
  }
  CUDA_TRY(cudaLaunchKernelEx(&cfg, kern, (const k::WaveStrand*)S.d_wave_strands, S.d_wave_data, bw, xs, g, st, tr));
  return {SPTRSV_SUCCESS, ""};
}

template <typename T, int K, int E>
Error launch_wave_e(Plan& p, Segment& S, const T* bw, T* xs, k::SolveState st, cudaStream_t s) {
  const bool glb = S.wave_global > 0;
  if (S.wave_GPC == 6)
    return glb ? launch_wave_t<T, K, E, 6, true>(p, S, bw, xs, st, s) : launch_wave_t<T, K, E, 6, false>(p, S, bw, xs, st, s);
  return glb ? launch_wave_t<T, K, E, k::kWaveGpcBig, true>(p, S, bw, xs, st, s)
             : launch_wave_t<T, K, E, k::kWaveGpcBig, false>(p, S, bw, xs, st, s);
}

template <typename T, int K>
Error launch_wave_k(Plan& p, Segment& S, const T* bw, T* xs, k::SolveState st, cudaStream_t s) {
  switch (S.wave_E) {
    case 0: return launch_wave_e<T, K, 0>(p, S, bw, xs, st, s);
    case 1: return launch_wave_e<T, K, 1>(p, S, bw, xs, st, s);
    default: return launch_wave_e<T, K, 2>(p, S, bw, xs, st, s);
  }
}

template <typename T>
Error launch_wave(Plan& p, Segment& S, const T* bw, T* xs, k::SolveState st, cudaStream_t s) {
  switch (S.wave_K) {
    case 2: return launch_wave_k<T, 2>(p, S, bw, xs, st, s);
    case 4: return launch_wave_k<T, 4>(p, S, bw, xs, st, s);
    default: return launch_wave_k<T, 8>(p, S, bw, xs, st, s);
  }
}

// Cooperative launch of the static warp-per-item sync-free kernel: the grid
// is the co-resident maximum (all warps must be resident for the static
// schedule, see k::tri_sf_wrow), capped by the item count.
template <typename T>
Error launch_sf_wrow(Plan& p, Segment& S, int nitem, const T* val, const T* bw, T* xs, k::SolveState st,
                     cudaStream_t s) {
  auto kern = k::tri_sf_wrow<T, k::kSfWU>;
  static std::mutex mu;
  static std::unordered_map<int, int> per_sm_by_dev;
  int dev = 0;
  CUDA_TRY(cudaGetDevice(&dev));
  int per_sm = 0;
  {
    std::lock_guard<std::mutex> g(mu);
    auto it = per_sm_by_dev.find(dev);
    if (it == per_sm_by_dev.end()) {
      CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 256, 0));
      per_sm_by_dev[dev] = per_sm;
    } else {
      per_sm = it->second;
    }
  }
  int nb = std::max(1, per_sm) * p.sm_count;
  if (const char* e = std::getenv("SPTRSV_SF_WROW_CTAS")) nb = std::min(nb, std::max(1, std::atoi(e)));  // tuning
  nb = std::max(1, std::min<int>(nb, (int)cdiv(nitem, 8)));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(nb);
  cfg.blockDim = dim3(256);
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  CUDA_TRY(cudaLaunchKernelEx(&cfg, kern, S.info.row0, nitem, (const k::SfItem*)S.d_sf_items, S.d_ci, val, bw, xs,
                              (T*)p.d_part, st));
  return {SPTRSV_SUCCESS, ""};
}

// k::tri_level_cluster: one cluster of S.cl_size CTAs (non-portable above 8)
template <typename T>
Error launch_cluster(Plan& p, Segment& S, const T* bw, T* xs, k::SolveState st, cudaStream_t s) {
  auto kern = k::tri_level_cluster<T>;
  CUDA_TRY(ensure_smem_attr((const void*)kern, 0, S.cl_size > 8));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(S.cl_size);
  cfg.blockDim = dim3(SPTRSV_CL_NT);
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = S.cl_size;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  const int* ip = S.d_sf_items + (size_t)S.cl_nitem * 8;
  CUDA_TRY(cudaLaunchKernelEx(&cfg, kern, S.info.row0, S.info.nlevels, ip, (const k::SfItem*)S.d_sf_items, S.d_rp,
                              S.d_ci, (const T*)S.d_val, bw, xs, (T*)p.d_part, st));
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
      if (nrhs == 1 && S.fused) {
        // computed by the preceding triangle's kernel (fused trailing items)
      } else if (S.dev_nzr > 0 && I.nnz > 0) {
        const bool dcsr = S.dev_dcsr;
        if (nrhs == 1 && I.impl == SPTRSV_IMPL_SQ_ADAPT) {
          const int nitem = (int)(S.sq_items.size() / 4);
          const auto* items = (const k::SqItem*)S.d_sq_items;
          unsigned g = cdiv(nitem, 8);
          if (dcsr)
            k::sq_adapt_1<T, true><<<g, 256, 0, s>>>(nitem, I.row0, items, S.d_rows, S.d_rp, S.d_ci, val, xs, bw);
          else
            k::sq_adapt_1<T, false><<<g, 256, 0, s>>>(nitem, I.row0, items, S.d_rows, S.d_rp, S.d_ci, val, xs, bw);
        } else if (nrhs == 1) {
          if (I.impl == SPTRSV_IMPL_SQ_VECTOR) {
            unsigned g = cdiv((int64_t)S.dev_nzr * 32, 256);
            if (dcsr)
              k::sq_vector_1<T, true><<<g, 256, 0, s>>>(S.dev_nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs, bw);
            else
              k::sq_vector_1<T, false><<<g, 256, 0, s>>>(S.dev_nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs, bw);
          } else {
            unsigned g = cdiv(S.dev_nzr, 256);
            if (dcsr)
              k::sq_scalar_1<T, true><<<g, 256, 0, s>>>(S.dev_nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs, bw);
            else
              k::sq_scalar_1<T, false><<<g, 256, 0, s>>>(S.dev_nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs, bw);
          }
        } else if (nrhs >= 64 && (int64_t)(I.col1 - I.col0) * nrhs * (int64_t)sizeof(T) > (int64_t(64) << 20) &&
                   p.spmm.tile > 0) {
          // X rows of the square's columns exceed L2: RHS-tiled SpMM
          auto launch_tiled = [&](auto Gc) {
            constexpr int Gv = decltype(Gc)::value;
            const dim3 g(cdiv((int64_t)S.dev_nzr * Gv, 256), cdiv(nrhs, Gv));
            if (dcsr)
              k::sq_multi_tiled<T, Gv, 1, 2, true><<<g, 256, 0, s>>>(S.dev_nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val,
                                                                     xs, bw, nrhs);
            else
              k::sq_multi_tiled<T, Gv, 1, 2, false><<<g, 256, 0, s>>>(S.dev_nzr, I.row0, S.d_rows, S.d_rp, S.d_ci,
                                                                      val, xs, bw, nrhs);
          };
          if (p.spmm.tile == 8)
            launch_tiled(std::integral_constant<int, 8>());
          else if (p.spmm.tile == 16)
            launch_tiled(std::integral_constant<int, 16>());
          else
            launch_tiled(std::integral_constant<int, 32>());
        } else {
          dispatch_multi_un(nrhs, p.spmm, [&](auto G, auto R, auto U) {
            unsigned g = cdiv((int64_t)S.dev_nzr * G, 256);
            if (dcsr)
              k::sq_multi<T, G, R, U, true><<<g, 256, 0, s>>>(S.dev_nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs,
                                                              bw, nrhs);
            else
              k::sq_multi<T, G, R, U, false><<<g, 256, 0, s>>>(S.dev_nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs,
                                                               bw, nrhs);
          });
        }
      }
    } else if (m > 0) {  // triangle: x_seg = L_seg^{-1} b_seg
      switch (I.impl) {
        case SPTRSV_IMPL_TRI_DIAG:
          k::tri_diag<T><<<cdiv((int64_t)m * nrhs, 256), 256, 0, s>>>(I.row0, m, nrhs, bw, xs);
          break;
        case SPTRSV_IMPL_TRI_SYNCFREE:
          // B200: a few-level triangle with several RHS runs level by level
          // (bandwidth-bound launches; the level-set label's own kernel)
          if (!(nrhs > 1 && p.opts.selector == SPTRSV_SELECT_B200 && p.reorder_eff == 0 && I.nlevels <= 20))
            goto sync_free;
          [[fallthrough]];
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
              dispatch_multi_un(nrhs, p.spmm, [&](auto G, auto R, auto U) {
                k::tri_level_multi<T, G, R, U><<<cdiv((int64_t)(rb - ra) * G, 256), 256, 0, s>>>(
                    ra, rb, I.row0, S.d_rp, S.d_ci, val, bw, xs, nrhs);
              });
            }
          }
          break;
        }
        case SPTRSV_IMPL_TRI_PIPE:
          if (nrhs == 1 && S.wave_K > 0) {
            Error e = launch_wave<T>(p, S, bw, xs, st, s);
            if (e.status) return e;
          } else {  // nrhs > 1: the device row order is not level-contiguous; the
                    // multi-RHS sync-free kernel runs on the execution-order CSR
            dispatch_multi(nrhs, [&](auto G, auto R) {
              k::tri_syncfree_multi<T, G, R><<<std::max(1u, std::min<unsigned>(cdiv(m, 256 / G), p.sm_count * 2)),
                                               256, 0, s>>>(I.row0, m, S.d_rp, S.d_ci, val, bw, xs, st,
                                                            S.ticket_slot, nrhs);
            });
          }
          break;
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
            CUDA_TRY(ensure_smem_attr((const void*)k::tri_chain_tma<T>, smem, false));
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
            dispatch_multi_un(nrhs, p.spmm, [&](auto G, auto R, auto U) {
              k::tri_chain_multi<T, G, R, U><<<1, 1024, 0, s>>>(I.row0, I.nlevels, S.d_level_ptr, S.d_rp, S.d_ci,
                                                            val, bw, xs, nrhs);
            });
          }
          break;
        }
        case SPTRSV_IMPL_TRI_SUPERNODE:
          if (nrhs == 1) {
            const int nit = (int)(S.sn_items.size() / 8);
            const unsigned g = std::max(1u, std::min<unsigned>(cdiv(nit, 8), p.sm_count * 8));
            k::tri_supernode<T><<<g, 256, 0, s>>>(nit, (const k::SnItem*)S.d_sn_items, (const k::SnDesc*)S.d_sn_desc,
                                                  S.d_sn_cols, (const T*)S.d_sn_vals, (const T*)S.d_sn_blk, bw, xs,
                                                  (T*)p.d_part + S.sn_part_base, st, S.ticket_slot);
            break;
          }
          if (nrhs >= kSnMultiMinRhs && !std::getenv("SPTRSV_NO_SN_MULTI")) {
            const int np = (int)S.sn_ptr.size() - 1;
            const unsigned g = std::max(1u, std::min<unsigned>(np, p.sm_count * 4));
            // one launch per 64-column chunk: inside a launch a piece's
            // chunks would run one after the other on the elimination-tree
            // chain; as separate launches each chain is one chunk long.
            // Launch i polls and publishes epoch + i and reclaims pieces from
            // a re-zeroed ticket.
            const int nch = (int)cdiv(nrhs, k::kSnmCols);
            for (int c = 0; c < nch; ++c) {
              k::SolveState sc = st;
              sc.epoch_off = (uint32_t)c;
              if (c > 0) CUDA_TRY(cudaMemsetAsync(st.tickets + S.ticket_slot, 0, 4, s));
              k::tri_supernode_multi<T><<<g, 256, 0, s>>>(np, (const k::SnDesc*)S.d_sn_desc, S.d_sn_cols,
                                                          (const T*)S.d_sn_vals, (const T*)S.d_sn_blk, bw, xs, sc,
                                                          S.ticket_slot, nrhs, c * k::kSnmCols,
                                                          std::min(nrhs, (c + 1) * k::kSnmCols));
            }
            break;
          }
          [[fallthrough]];  // 1 < nrhs < 16: the multi-RHS sync-free kernel on the CSR copy
        sync_free:
        default: {  // SPTRSV_IMPL_TRI_SYNCFREE
          // enough resident warps for about two of the triangle's widest
          // levels: more only spin on rows whose dependencies are levels away
          const int cap = p.sm_count * 8;  // 8 CTAs x 8 warps per SM
          const int64_t wl = std::max<int64_t>(1, I.max_level_rows);
          // (round-1 sweeps on C3: 2 CTAs/SM best for thread-per-row, 3 for
          // warp-per-row; the full 8/SM grid was 1.5x slower)
          auto ctas = [&](int64_t rows_per_cta, int64_t rows_total) {
            const int per_sm = rows_per_cta == 8 ? 3 : 2;
            int64_t c = std::max<int64_t>((int64_t)per_sm * p.sm_count, cdiv(2 * wl, rows_per_cta));
            if (rows_per_cta == 8) c = (int64_t)per_sm * p.sm_count;
            if (const char* ev2 = std::getenv("SPTRSV_SF_CTAS")) c = std::max(1, std::atoi(ev2));
            return (unsigned)std::min<int64_t>({c, (int64_t)cap, (int64_t)cdiv(rows_total, rows_per_cta)});
          };
          if (nrhs == 1 && S.cl_size > 0) {
            Error e = launch_cluster<T>(p, S, bw, xs, st, s);
            if (e.status) return e;
          } else if (nrhs == 1 && !S.sf_items.empty()) {
            const int nitem = (int)(S.sf_items.size() / 8);
            int nctas = SPTRSV_SF_MINB * p.sm_count;
            if (const char* e2 = std::getenv("SPTRSV_SF_CTAS")) nctas = std::max(1, std::atoi(e2));  // tuning
            const unsigned g = std::max(1u, std::min<unsigned>(cdiv(nitem, 8), (unsigned)nctas));
            if (S.sf_wrow) {
              Error e2 = launch_sf_wrow<T>(p, S, nitem, val, bw, xs, st, s);
              if (e2.status) return e2;
            } else if (S.sf_mixed) {
              k::SqDesc sq{nullptr, nullptr, nullptr, nullptr, 0, 0};
              if (S.fused_sq >= 0) {
                const Segment& Q = p.segs[S.fused_sq];
                sq = k::SqDesc{Q.d_rows, Q.d_rp, Q.d_ci, Q.d_val, Q.info.row0, Q.dev_dcsr ? 1 : 0};
              }
              k::tri_sf_mixed<T, SPTRSV_SF_U><<<std::max(1u, ctas(256, m)), 256, 0, s>>>(
                  I.row0, nitem, (const k::SfItem*)S.d_sf_items, S.d_rp, S.d_ci, val, bw, xs, (T*)p.d_part, st,
                  S.ticket_slot, sq);
            }
            else
              k::tri_sf_items<T><<<g, 256, 0, s>>>(I.row0, nitem, (const k::SfItem*)S.d_sf_items, S.d_rp, S.d_ci,
                                                   val, bw, xs, (T*)p.d_part, st, S.ticket_slot);
          } else if (nrhs == 1) {
            if (tri_use_warp(S))
              k::tri_syncfree_warp<T, 8><<<std::max(1u, ctas(8, m)), 256, 0, s>>>(I.row0, m, S.d_rp, S.d_ci, val,
                                                                                  bw, xs, st, S.ticket_slot);
            else
              k::tri_syncfree_thread<T, 4, 32><<<std::max(1u, ctas(256, m)), 256, 0, s>>>(
                  I.row0, m, S.d_rp, S.d_ci, val, bw, xs, st, S.ticket_slot);
          } else {
            dispatch_multi(nrhs, [&](auto G, auto R) {
              k::tri_syncfree_multi<T, G, R><<<std::max(1u, ctas(256 / G, m)), 256, 0, s>>>(
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
      c += (S.nzr > 0 && S.info.nnz > 0 && !S.fused);
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
    if (S.wave_K > 0) {  // raw per-strand stamps -> $SPTRSV_TRACE_DIR/wave_seg<i>.bin
      const size_t nt = (size_t)S.wave_C * S.wave_W * 1024;
      cudaMemcpy(S.h_trace.data(), S.d_trace, nt * 8, cudaMemcpyDeviceToHost);
      const char* dir = std::getenv("SPTRSV_TRACE_DIR");
      std::string path = std::string(dir ? dir : ".") + "/wave_seg" + std::to_string(si) + ".bin";
      if (FILE* f = std::fopen(path.c_str(), "wb")) {
        std::fwrite(S.h_trace.data(), 8, nt, f);
        std::fclose(f);
      }
      continue;
    }
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

// Epochs one solve hands out (multi-RHS sync-free triangles poll per-row
// flags holding the epoch of the solve that published them; the supernodal
// SpTRSM runs one launch per 64-column chunk, each with its own epoch).
uint32_t epoch_span(const Plan& p, int nrhs) {
  if (nrhs <= 1 || !p.needs_flags) return 0;
  return (uint32_t)std::max<int64_t>(1, cdiv(nrhs, k::kSnmCols));
}

void drop_graphs(Plan& p) {
  for (auto& g : p.graphs)
    if (g.exec) cudaGraphExecDestroy((cudaGraphExec_t)g.exec);
  p.graphs.clear();
  p.pending = GraphEntry{};
}

// Everything a solve of nrhs columns needs that is not a kernel launch:
// workspace, flags, epoch wrap.  Runs before (never inside) a graph capture.
Error prepare_solve(Plan& p, int nrhs, cudaStream_t s) {
  const int n = p.n;
  const size_t need = (size_t)n * nrhs * p.vbytes;
  if (need > p.ws.w_bytes) {
    drop_graphs(p);  // captured solves reference the old workspace
    dfree(p, p.ws.bw, s);
    dfree(p, p.ws.xs, s);
    p.ws.bw = p.ws.xs = nullptr;
    p.ws.w_bytes = 0;
    // +256 B: the staged chain kernel's 16-byte-aligned TMA windows may read
    // up to 15 bytes past the last row
    p.ws.bw = dalloc(p, need + 256, s);
    p.ws.xs = dalloc(p, need + 256, s);
    if (!p.ws.bw || !p.ws.xs) return {SPTRSV_ERROR_ALLOC, "workspace allocation failed"};
    p.ws.w_bytes = need;
  }
  const uint32_t span = epoch_span(p, nrhs);
  if (span) {
    if (!p.ws.flags) {
      drop_graphs(p);
      p.ws.flags_n = std::max(1, n);
      p.ws.flags = dalloc(p, (size_t)p.ws.flags_n * 4, s);
      if (!p.ws.flags) return {SPTRSV_ERROR_ALLOC, "flag workspace allocation failed"};
      CUDA_TRY(cudaMemsetAsync(p.ws.flags, 0, (size_t)p.ws.flags_n * 4, s));
      CUDA_TRY(cudaMemsetAsync(p.d_epoch, 0, 8, s));
      p.epoch = 0;
    }
    // the device counter is mirrored here: about to wrap -> restart from
    // clean flags (stream-ordered, before the solve that would wrap)
    if (p.epoch > 0xFFFFFFFFu - span - 1u) {
      CUDA_TRY(cudaMemsetAsync(p.ws.flags, 0, (size_t)p.ws.flags_n * 4, s));
      CUDA_TRY(cudaMemsetAsync(p.d_epoch, 0, 8, s));
      p.epoch = 0;
    }
    p.epoch += span;
  }
  return {SPTRSV_SUCCESS, ""};
}

// The kernels of one solve (permute-in, Alg 7's segment loop, permute-out)
// enqueued on s; no allocation, no host synchronisation (capturable).
template <typename T>
Error solve_device(Plan& p, const T* b, int64_t ldb, T* x, int64_t ldx, int nrhs, sptrsv_layout_t layout,
                   cudaStream_t s) {
  const int n = p.n;
  T* bw = (T*)p.ws.bw;
  T* xs = (T*)p.ws.xs;
  const T* rd = (const T*)p.d_rdiag;
  // nrhs == 1: sync-free rows poll their dependencies' values, which start
  // as the sentinel; nrhs > 1: they poll per-row epoch flags instead
  const int fill = (p.needs_sentinel && nrhs == 1) ? 1 : 0;
  if (const char* e = std::getenv("SPTRSV_SF_BACKOFF")) p.backoff_ns = (uint32_t)std::max(0, std::atoi(e));  // tuning
  k::SolveState st{p.d_tickets,         p.nticket,    p.d_error, (uint32_t*)p.ws.flags, p.d_epoch, 0u,
                   epoch_span(p, nrhs), p.backoff_ns, p.d_derr,  p.wd_spins, (unsigned long long*)p.d_sf_trace};
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
    k::perm_in_1<T><<<std::max(1u, cdiv(std::max(n, p.npart), 256)), 256, 0, s>>>(n, p.d_perm, rd, b, stride, bw, xs,
                                                                                  fill, st, (T*)p.d_part, p.npart);
  } else if (layout == SPTRSV_COL_MAJOR) {
    k::perm_in_cm<T><<<std::max(1u, cdiv(n, 32)), 256, 0, s>>>(n, nrhs, iperm, rd, b, ldb, bw, xs, fill, st);
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
    k::perm_out_cm<T><<<std::max(1u, cdiv(n, 32)), 256, 0, s>>>(n, nrhs, iperm, xs, x, ldx);
  } else {
    k::perm_out_rm<T><<<std::max(1u, cdiv((int64_t)n * nrhs, 256)), 256, 0, s>>>(n, nrhs, p.d_perm, xs, x, ldx);
  }
  CUDA_TRY(cudaGetLastError());
  if (ev) {
    CUDA_TRY(cudaEventRecord(ev[2 + p.segs.size()], s));
    p.last_nseg_timed = (int)p.segs.size();
  }
  if (p.trace) dump_trace(p, s);
  if (p.d_sf_trace) {  // debug: the last solve's per-row stamps -> $SPTRSV_SF_TRACE/sf_trace.bin
    cudaStreamSynchronize(s);
    std::vector<unsigned long long> h((size_t)n * 2);
    cudaMemcpy(h.data(), p.d_sf_trace, h.size() * 8, cudaMemcpyDeviceToHost);
    std::string path = std::string(std::getenv("SPTRSV_SF_TRACE")) + "/sf_trace.bin";
    if (FILE* f = std::fopen(path.c_str(), "wb")) {
      std::fwrite(h.data(), 8, h.size(), f);
      std::fclose(f);
    }
    cudaMemsetAsync(p.d_sf_trace, 0, h.size() * 8, s);
  }
  return {SPTRSV_SUCCESS, ""};
}

// prepare + enqueue (the host-pointer paths)
Error solve_device_any(Plan& p, const void* b, int64_t ldb, void* x, int64_t ldx, int nrhs, sptrsv_layout_t layout,
                       cudaStream_t s) {
  Error e = prepare_solve(p, nrhs, s);
  if (e.status) return e;
  return p.dtype == SPTRSV_R64F
             ? solve_device<double>(p, (const double*)b, ldb, (double*)x, ldx, nrhs, layout, s)
             : solve_device<float>(p, (const float*)b, ldb, (float*)x, ldx, nrhs, layout, s);
}

// memory type (0 host / unregistered, 1 device or managed) and device ordinal
int ptr_kind(const void* ptr, int* device) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, ptr) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  *device = a.device;
  return (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) ? 1 : 0;
}

}  // namespace

// Work items of the row-block square kernel (k::sq_adapt_1): greedy runs of
// <= 32 consecutive stored rows with <= kSqNB entries; a longer row is an
// item of its own, cut into kSqLW-entry chunks (flagged: atomic update) when
// longer than kSqLW.
void build_sq_items(Segment& S) {
  S.sq_items.clear();
  const auto& I = S.info;
  if (I.kind != 1 || I.impl != SPTRSV_IMPL_SQ_ADAPT || S.nzr == 0) return;
  const int nzr = S.nzr;
  const std::vector<int32_t>& rp = S.rp;
  auto push = [&](int t0, int t1, int p0, int p1, bool split) {
    S.sq_items.push_back(t0);
    S.sq_items.push_back(split ? (int32_t)((uint32_t)t1 | 0x80000000u) : t1);
    S.sq_items.push_back(p0);
    S.sq_items.push_back(p1);
  };
  int t = 0;
  while (t < nzr) {
    const int len = rp[t + 1] - rp[t];
    if (len > k::kSqNB) {
      if (len <= k::kSqLW) {
        push(t, t + 1, rp[t], rp[t + 1], false);
      } else {
        for (int p0 = rp[t]; p0 < rp[t + 1]; p0 += k::kSqLW)
          push(t, t + 1, p0, std::min(p0 + k::kSqLW, rp[t + 1]), true);
      }
      ++t;
      continue;
    }
    const int start = t;
    int tot = 0;
    while (t < nzr && t - start < 32 && tot + (rp[t + 1] - rp[t]) <= k::kSqNB) {
      tot += rp[t + 1] - rp[t];
      ++t;
    }
    push(start, t, rp[start], rp[t], false);
  }
}

// Work items of the row-block sync-free kernel (k::tri_sf_items): greedy
// runs of <= 32 consecutive rows holding <= kSfNB off-diagonal entries; a
// longer row is cut into kSfNB-entry pieces (kind 1, each with a partial-sum
// slot out of the plan's `part` array) closed by its last piece (kind 2),
// which adds the earlier pieces' partial sums.  SPTRSV_SF_V1 keeps the
// round-1 kernels (thread / warp per row).
void build_sf_mixed(Segment& S, int32_t& part_base);
// Fuse square Q (the next segment) into triangle T's mixed sync-free kernel
// as trailing items (k::tri_sf_mixed kinds 4 / 5): greedy blocks of <= 32
// stored rows holding <= kSfNB entries; a longer row in kSfNB-entry chunks
// (atomic updates).  Items index Q's DEVICE row structure (Q.rp, with
// Q.dev_dcsr / d_rows mapping stored row -> row).
void fuse_square_items(Segment& T, Segment& Q) {
  if (Q.info.kind != 1 || Q.info.nnz == 0 || Q.dev_nzr == 0) return;
  const std::vector<int32_t>& rp = Q.rp;
  const int nzr = Q.dev_nzr;
  auto push = [&](int t0, int t1, int p0, int p1, int kind) {
    const int32_t rec[8] = {t0, t1, p0, p1, kind, 0, 0, 0};
    T.sf_items.insert(T.sf_items.end(), rec, rec + 8);
  };
  int t = 0;
  while (t < nzr) {
    const int len = rp[t + 1] - rp[t];
    if (len > k::kSfNB) {
      for (int a = rp[t]; a < rp[t + 1]; a += k::kSfNB) push(t, t + 1, a, std::min(a + k::kSfNB, rp[t + 1]), 5);
      ++t;
      continue;
    }
    const int start = t;
    int tot = 0;
    while (t < nzr && t - start < 32 && tot + (rp[t + 1] - rp[t]) <= k::kSfNB) {
      tot += rp[t + 1] - rp[t];
      ++t;
    }
    push(start, t, rp[start], rp[t], 4);
  }
  Q.fused = true;
}

// Items of the static warp-per-item kernel (k::tri_sf_wrow): one per row of
// <= kSfW entries, else kSfW-entry pieces closed by the row's last piece.
void build_sf_wrow(Segment& S, int32_t& part_base) {
  const auto& I = S.info;
  const int m = I.row1 - I.row0;
  const std::vector<int32_t>& rp = S.rp;
  S.sf_items.reserve((size_t)m * 8);
  for (int t = 0; t < m; ++t) {
    const int len = rp[t + 1] - rp[t];
    const int np = std::max(1, (len + k::kSfW - 1) / k::kSfW);
    const int first = part_base;
    for (int q = 0; q < np; ++q) {
      const int a = rp[t] + q * k::kSfW, b = std::min(a + k::kSfW, rp[t + 1]);
      const int kind = np == 1 ? 0 : (q < np - 1 ? 1 : 2);
      const int32_t rec[8] = {t, t + 1, a, b, kind, kind == 1 ? part_base++ : first, kind == 2 ? part_base : 0, 0};
      S.sf_items.insert(S.sf_items.end(), rec, rec + 8);
    }
  }
}
// Items of the cluster level-set kernel (k::tri_level_cluster): the
// tri_sf_mixed kinds, cut at level boundaries, then ip[nlevels + 1] (first
// item of every level) appended to the same array.
void build_cl_items(Segment& S, int32_t& part_base, int cs) {
  const auto& I = S.info;
  const std::vector<int32_t>& rp = S.rp;
  const std::vector<int32_t>& lp = S.level_ptr;
  auto push = [&](int t0, int t1, int p0, int p1, int kind, int s0, int s1) {
    const int32_t rec[8] = {t0, t1, p0, p1, kind, s0, s1, 0};
    S.sf_items.insert(S.sf_items.end(), rec, rec + 8);
  };
  std::vector<int32_t> ip(I.nlevels + 1, 0);
  for (int l = 0; l < I.nlevels; ++l) {
    ip[l] = (int32_t)(S.sf_items.size() / 8);
    int t = lp[l];
    const int tend = lp[l + 1];
    while (t < tend) {
      const int len = rp[t + 1] - rp[t];
      if (len > k::kSfLong) {
        if (len <= k::kSfNB) {
          push(t, t + 1, rp[t], rp[t + 1], 3, 0, 0);
        } else {
          const int np = (len + k::kSfNB - 1) / k::kSfNB;
          const int first = part_base;
          for (int q = 0; q < np; ++q) {
            const int a = rp[t] + q * k::kSfNB, b = std::min(a + k::kSfNB, rp[t + 1]);
            if (q < np - 1)
              push(t, t + 1, a, b, 1, part_base++, 0);
            else
              push(t, t + 1, a, b, 2, first, part_base);
          }
        }
        ++t;
        continue;
      }
      const int start = t;
      while (t < tend && t - start < 32 && rp[t + 1] - rp[t] <= k::kSfLong) ++t;
      push(start, t, rp[start], rp[t], 0, 0, 0);
    }
  }
  ip[I.nlevels] = (int32_t)(S.sf_items.size() / 8);
  S.cl_nitem = ip[I.nlevels];
  S.sf_items.insert(S.sf_items.end(), ip.begin(), ip.end());
  S.cl_size = cs;
}

void build_sf_items(Segment& S, int32_t& part_base, int selector) {
  S.sf_items.clear();
  S.sf_mixed = S.sf_wrow = false;
  S.cl_size = 0;
  S.cl_nitem = 0;
  const auto& I = S.info;
  if (I.kind != 0 || I.impl != SPTRSV_IMPL_TRI_SYNCFREE || selector != SPTRSV_SELECT_B200) return;
  if (const char* e = std::getenv("SPTRSV_SF_CLUSTER")) {  // experiment: level-set on one cluster
    const int cs = std::atoi(e);
    if (cs >= 1 && cs <= 16 && (int)S.level_ptr.size() == I.nlevels + 1 && I.nlevels > 1)
      return build_cl_items(S, part_base, cs);
  }
  // default (B200): the mixed-granularity kernel; SPTRSV_SF_V1 = the round-1
  // thread / warp-per-row kernels (kept for comparison)
  S.sf_mixed = std::getenv("SPTRSV_SF_V1") == nullptr && std::getenv("SPTRSV_SF_WROW") == nullptr &&
               std::getenv("SPTRSV_SF_ITEMS") == nullptr;
  if (S.sf_mixed) return build_sf_mixed(S, part_base);
  S.sf_wrow = std::getenv("SPTRSV_SF_WROW") != nullptr;
  if (S.sf_wrow) return build_sf_wrow(S, part_base);
  if (!std::getenv("SPTRSV_SF_ITEMS")) return;
  const int m = I.row1 - I.row0;
  const std::vector<int32_t>& rp = S.rp;
  auto push = [&](int t0, int t1, int p0, int p1, int kind, int s0, int s1) {
    const int32_t rec[8] = {t0, t1, p0, p1, kind, s0, s1, 0};
    S.sf_items.insert(S.sf_items.end(), rec, rec + 8);
  };
  int t = 0;
  while (t < m) {
    const int len = rp[t + 1] - rp[t];
    if (len > k::kSfNB) {
      const int np = (len + k::kSfNB - 1) / k::kSfNB;
      const int first = part_base;
      for (int q = 0; q < np; ++q) {
        const int a = rp[t] + q * k::kSfNB, b = std::min(a + k::kSfNB, rp[t + 1]);
        if (q < np - 1)
          push(t, t + 1, a, b, 1, part_base++, 0);
        else
          push(t, t + 1, a, b, 2, first, part_base);
      }
      ++t;
      continue;
    }
    const int start = t;
    int tot = 0;
    while (t < m && t - start < 32 && tot + (rp[t + 1] - rp[t]) <= k::kSfNB) {
      tot += rp[t + 1] - rp[t];
      ++t;
    }
    push(start, t, rp[start], rp[t], 0, 0, 0);
  }
}

// Work items of the mixed-granularity sync-free kernel (k::tri_sf_mixed):
// runs of <= 32 consecutive rows with <= kSfLong entries each (kind 0); a
// longer row is one warp item (kind 3) up to kSfNB entries, else kSfNB-entry
// pieces (kind 1) closed by its last piece (kind 2) with partial-sum slots.
void build_sf_mixed(Segment& S, int32_t& part_base) {
  const auto& I = S.info;
  const int m = I.row1 - I.row0;
  const std::vector<int32_t>& rp = S.rp;
  auto push = [&](int t0, int t1, int p0, int p1, int kind, int s0, int s1) {
    const int32_t rec[8] = {t0, t1, p0, p1, kind, s0, s1, 0};
    S.sf_items.insert(S.sf_items.end(), rec, rec + 8);
  };
  int t = 0;
  while (t < m) {
    const int len = rp[t + 1] - rp[t];
    if (len > k::kSfLong) {
      if (len <= k::kSfNB) {
        push(t, t + 1, rp[t], rp[t + 1], 3, 0, 0);
      } else {
        const int np = (len + k::kSfNB - 1) / k::kSfNB;
        const int first = part_base;
        for (int q = 0; q < np; ++q) {
          const int a = rp[t] + q * k::kSfNB, b = std::min(a + k::kSfNB, rp[t + 1]);
          if (q < np - 1)
            push(t, t + 1, a, b, 1, part_base++, 0);
          else
            push(t, t + 1, a, b, 2, first, part_base);
        }
      }
      ++t;
      continue;
    }
    const int start = t;
    while (t < m && t - start < 32 && rp[t + 1] - rp[t] <= k::kSfLong) ++t;
    push(start, t, rp[start], rp[t], 0, 0, 0);
  }
}

// Host -> device upload of the plan through pinned staging: pageable
// cudaMemcpy runs at a fraction of PCIe / C2C bandwidth, so large pieces are
// copied (in parallel) into one of two pinned 32 MB buffers, each sent with
// an async copy while the other is being filled.  Small pieces go directly.
struct PinnedStager {
  static constexpr size_t kBuf = size_t(32) << 20;
  char* buf[2] = {nullptr, nullptr};
  cudaEvent_t ev[2] = {nullptr, nullptr};
  int cur = 0;
  bool ok = false;
  cudaStream_t s = nullptr;
  PinnedStager() {
    ok = cudaHostAlloc((void**)&buf[0], kBuf, cudaHostAllocDefault) == cudaSuccess &&
         cudaHostAlloc((void**)&buf[1], kBuf, cudaHostAllocDefault) == cudaSuccess &&
         cudaEventCreateWithFlags(&ev[0], cudaEventDisableTiming) == cudaSuccess &&
         cudaEventCreateWithFlags(&ev[1], cudaEventDisableTiming) == cudaSuccess;
    if (!ok) cudaGetLastError();
  }
  cudaError_t put(char* dst, const void* src, size_t bytes) {
    if (!bytes) return cudaSuccess;
    if (!ok || bytes < (size_t(1) << 20)) return cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, s);
    const char* sp = (const char*)src;
    for (size_t o = 0; o < bytes; o += kBuf) {
      const size_t nb = std::min(kBuf, bytes - o);
      cudaError_t e = cudaEventSynchronize(ev[cur]);  // the buffer's previous copy is done
      if (e != cudaSuccess) return e;
      char* b = buf[cur];
      par_for((int64_t)nb, 0, [&](int64_t a, int64_t z) { std::memcpy(b + a, sp + o + a, (size_t)(z - a)); },
              int64_t(4) << 20);
      e = cudaMemcpyAsync(dst + o, b, nb, cudaMemcpyHostToDevice, s);
      if (e != cudaSuccess) return e;
      e = cudaEventRecord(ev[cur], s);
      if (e != cudaSuccess) return e;
      cur ^= 1;
    }
    return cudaSuccess;
  }
};

// Pool of mapped pinned host words for the plans' spin-wait watchdogs: one
// 4 KB page per 1024 plans, allocated on demand, never returned to the driver.
namespace {
std::mutex wd_mu;
std::vector<std::pair<int32_t*, int32_t*>> wd_free;  // (host, device) of free words
}  // namespace
bool watchdog_word_acquire(int32_t** h, int32_t** d) {
  std::lock_guard<std::mutex> g(wd_mu);
  if (wd_free.empty()) {
    int32_t* page = nullptr;
    int32_t* dpage = nullptr;
    if (cudaHostAlloc((void**)&page, 4096, cudaHostAllocMapped) != cudaSuccess ||
        cudaHostGetDevicePointer((void**)&dpage, page, 0) != cudaSuccess) {
      cudaGetLastError();
      return false;
    }
    for (int i = 1023; i >= 0; --i) wd_free.push_back({page + i, dpage + i});
  }
  *h = wd_free.back().first;
  *d = wd_free.back().second;
  wd_free.pop_back();
  return true;
}
void watchdog_word_release(int32_t* h) {
  std::lock_guard<std::mutex> g(wd_mu);
  // the device alias of a mapped host word is fixed: recover it
  int32_t* d = nullptr;
  if (cudaHostGetDevicePointer((void**)&d, h, 0) != cudaSuccess) {
    cudaGetLastError();
    return;
  }
  wd_free.push_back({h, d});
}

Error upload(Plan& p, void* stream_v) {
  cudaStream_t s = (cudaStream_t)stream_v;
  const size_t vb = p.vbytes;
  const int n = p.n;
  PhaseClock clk;
  // ---- arena layout (one allocation, segments in execution order, L229) ----
  size_t off = 0;
  auto take = [&](size_t bytes) {
    size_t o = off;
    off = align_up(off + bytes, 256);
    return o;
  };
  size_t o_perm = take((size_t)2 * n * 4);  // perm (new->old) then iperm (old->new)
  size_t o_rdiag = take((size_t)n * vb);
  struct Offs { size_t rp, ci, val, rows, lp, st, er, ed, sd, sc, sv, sbk, ps, pd, pc, sq, sf, sni; };
  std::vector<Offs> so(p.segs.size());
  p.trace = std::getenv("SPTRSV_TRACE") != nullptr;
  p.spmm = spmm_cfg();
  p.backoff_ns = 128;
  p.wd_spins = k::kWatchdogSpins;
  if (std::getenv("SPTRSV_SF_TRACE") && !p.d_sf_trace)  // debug: per-row claim/done stamps (SF_TRACE builds)
    if (cudaMalloc(&p.d_sf_trace, (size_t)std::max(1, n) * 16) != cudaSuccess) p.d_sf_trace = nullptr;
  if (const char* e = std::getenv("SPTRSV_WATCHDOG_SPINS"))  // tests: trip the watchdog quickly
    p.wd_spins = (uint32_t)std::max(1024, std::atoi(e));
  const k::ChainGeom cg = chain_geometry(p);
  p.chain_geom[0] = cg.NST; p.chain_geom[1] = cg.RMAX; p.chain_geom[2] = cg.EMAX;
  p.chain_geom[3] = cg.XW; p.chain_geom[4] = cg.LMAX;
  p.nticket = 0;
  p.npart = 0;
  p.needs_sentinel = false;
  p.needs_flags = false;
  for (size_t i = 0; i < p.segs.size(); ++i) build_wave(p, p.segs[i], vb);  // may switch a segment to CHAIN
  clk.lap("upload: build_wave");
  // execution order of the rows on the device: identity except inside wave
  // triangles (strand-major, group-major); sigma: new (plan) index -> device row
  std::vector<int32_t> sigma;
  for (auto& S : p.segs)
    if (S.wave_K > 0) {
      if (sigma.empty()) {
        sigma.resize(n);
        std::iota(sigma.begin(), sigma.end(), 0);
      }
      for (size_t q2 = 0; q2 < S.wave_tau.size(); ++q2) sigma[S.info.row0 + S.wave_tau[q2]] = S.info.row0 + (int)q2;
    }
  auto sg = [&](int32_t k2) { return sigma.empty() ? k2 : sigma[k2]; };
  // device images of the segment CSR in device row order: views of the
  // segment's own arrays, or owned re-ordered copies where sigma moves rows
  struct Dev {
    std::vector<int32_t> rp_o, rows_o;
    dvec<int32_t> ci_o;
    dvec<char> val_o;
    const int32_t *rp = nullptr, *ci = nullptr, *rows = nullptr;
    const char* val = nullptr;
    size_t nrp = 0, nci = 0, nrows = 0, nval = 0;
  };
  std::vector<Dev> dv(p.segs.size());
  for (size_t i = 0; i < p.segs.size(); ++i) {
    Segment& S = p.segs[i];
    Dev& D = dv[i];
    const auto& I = S.info;
    if (I.kind == 0 && S.wave_K > 0) {  // rows permuted by wave_tau
      const int m = I.row1 - I.row0;
      D.rp_o.assign(m + 1, 0);
      D.ci_o.reserve(S.ci.size());
      D.val_o.reserve(S.val.size());
      for (int q2 = 0; q2 < m; ++q2) {
        const int r = S.wave_tau[q2];
        for (int e = S.rp[r]; e < S.rp[r + 1]; ++e) D.ci_o.push_back(sg(S.ci[e]));
        D.val_o.insert(D.val_o.end(), S.val.begin() + (size_t)S.rp[r] * vb, S.val.begin() + (size_t)S.rp[r + 1] * vb);
        D.rp_o[q2 + 1] = (int32_t)D.ci_o.size();
      }
      D.rp = D.rp_o.data(); D.nrp = D.rp_o.size();
      D.ci = D.ci_o.data(); D.nci = D.ci_o.size();
      D.val = D.val_o.data(); D.nval = D.val_o.size();
    } else {
      D.rp = S.rp.data(); D.nrp = S.rp.size();
      D.val = S.val.data(); D.nval = S.val.size();
      if (!sigma.empty()) {
        D.ci_o.resize(S.ci.size());
        for (size_t q2 = 0; q2 < S.ci.size(); ++q2) D.ci_o[q2] = sigma[S.ci[q2]];
        D.ci = D.ci_o.data();
      } else {
        D.ci = S.ci.data();
      }
      D.nci = S.ci.size();
    }
    S.dev_dcsr = I.kind == 1 && I.format == SPTRSV_FMT_DCSR;
    S.dev_nzr = S.nzr;
    D.rows = S.rows.data();
    D.nrows = S.rows.size();
    if (I.kind == 1) {
      if (S.dev_dcsr) {
        if (!sigma.empty()) {
          D.rows_o = S.rows;
          for (auto& r : D.rows_o) r = sg(r);
          D.rows = D.rows_o.data();
        }
      } else {
        bool moved = false;
        for (int r = I.row0; r < I.row1 && !sigma.empty() && !moved; ++r) moved = sigma[r] != r;
        if (moved) {  // CSR rows reordered: upload as DCSR with every row listed
          S.dev_dcsr = true;
          D.rows_o.resize(I.row1 - I.row0);
          for (int r = I.row0; r < I.row1; ++r) D.rows_o[r - I.row0] = sigma[r];
          D.rows = D.rows_o.data();
          D.nrows = D.rows_o.size();
          S.dev_nzr = I.row1 - I.row0;
        }
      }
    }
  }
  for (auto& S : p.segs) S.fused = false;
  for (size_t i = 0; i < p.segs.size(); ++i) {
    Segment& S = p.segs[i];
    build_chain_stages(S, cg);
    build_chain_ell(S, vb);
    build_supernodes(S, vb, p.npart);
    build_sq_items(S);
    build_sf_items(S, p.npart, p.opts.selector);
    S.fused_sq = -1;
    if (S.sf_mixed && i + 1 < p.segs.size() && std::getenv("SPTRSV_SQ_FUSE")) {
      fuse_square_items(S, p.segs[i + 1]);
      if (p.segs[i + 1].fused) S.fused_sq = (int)i + 1;
    }
    so[i].er = take(S.ell_recs.size() * 4);
    so[i].ed = take(S.ell_data.size());
    so[i].rp = take(dv[i].nrp * 4);
    so[i].ci = take(dv[i].nci * 4);
    so[i].val = take(dv[i].nval);
    so[i].rows = take(dv[i].nrows * 4);
    so[i].lp = take(S.level_ptr.size() * 4);
    so[i].st = take(S.chain_recs.size() * 4);
    so[i].sd = take(S.sn_desc.size());
    so[i].sc = take(S.sn_cols.size() * 4);
    so[i].sv = take(S.sn_vals.size());
    so[i].sbk = take(S.sn_blk.size());
    so[i].ps = take(S.wave_strands.size());
    so[i].pd = take(S.wave_data.size());
    so[i].pc = take(S.wave_crows.size() * 4);
    so[i].sq = take(S.sq_items.size() * 4);
    so[i].sf = take(S.sf_items.size() * 4);
    so[i].sni = take(S.sn_items.size() * 4);
    if (S.info.kind == 0) S.ticket_slot = p.nticket++;
    if (S.info.kind == 0 && (S.info.impl == SPTRSV_IMPL_TRI_SYNCFREE || S.info.impl == SPTRSV_IMPL_TRI_SUPERNODE ||
                             (S.info.impl == SPTRSV_IMPL_TRI_PIPE && (S.wave_K == 0 || S.wave_global > 0))))
      p.needs_sentinel = true;
    if (S.info.kind == 0 && (S.info.impl == SPTRSV_IMPL_TRI_SYNCFREE || S.info.impl == SPTRSV_IMPL_TRI_SUPERNODE ||
                             S.info.impl == SPTRSV_IMPL_TRI_PIPE))
      p.needs_flags = true;
  }
  size_t o_tickets = take((size_t)std::max(1, p.nticket) * 4);
  size_t o_ctl = take(16);  // {watchdog word, pad, epoch base, last epoch}
  size_t o_part = take((size_t)std::max(1, p.npart) * vb);
  p.arena_bytes = off;
  clk.lap("upload: chain/ell/supernode");

  int dev;
  CUDA_TRY(cudaGetDevice(&dev));
  p.device = dev;
  p.arena = dalloc(p, std::max<size_t>(off, 256), s);
  if (!p.arena) return {SPTRSV_ERROR_ALLOC, "plan arena allocation failed (" + std::to_string(off) + " bytes)"};
  clk.lap("upload: cudaMalloc");
  // perm / iperm / 1/d are composed on the host (sigma), every segment array
  // is copied straight from its host vector (no staging image of the arena)
  std::vector<char> h(o_rdiag + (size_t)n * vb, 0);
  // p.perm is in ORIGINAL indexing (UPPER: composed with J); the device
  // gathers b[perm_dev[k]] into device row k and scatters x back
  {
    int32_t* pd = (int32_t*)&h[o_perm];
    int32_t* ip = pd + n;
    char* rd = &h[o_rdiag];
    for (int k2 = 0; k2 < n; ++k2) {
      const int d = sg(k2);
      pd[d] = p.perm[k2];
      ip[p.perm[k2]] = d;
      std::memcpy(rd + (size_t)d * vb, &p.rdiag_new[(size_t)k2 * vb], vb);
    }
  }
  char* A = (char*)p.arena;
  CUDA_TRY(cudaMemsetAsync(A, 0, off, s));  // padding and tickets
  CUDA_TRY(cudaMemcpyAsync(A, h.data(), h.size(), cudaMemcpyHostToDevice, s));
  // one stager per process (pinned buffers are costly to allocate), used
  // by one upload at a time
  static std::mutex stager_mu;
  static PinnedStager* stager = nullptr;
  std::lock_guard<std::mutex> stager_lock(stager_mu);
  if (!stager) stager = new PinnedStager();
  stager->s = s;
  auto put = [&](size_t o, const void* src, size_t bytes) -> cudaError_t { return stager->put(A + o, src, bytes); };
  for (size_t i = 0; i < p.segs.size(); ++i) {
    Segment& S = p.segs[i];
    const Dev& D = dv[i];
    CUDA_TRY(put(so[i].rp, D.rp, D.nrp * 4));
    CUDA_TRY(put(so[i].ci, D.ci, D.nci * 4));
    CUDA_TRY(put(so[i].val, D.val, D.nval));
    CUDA_TRY(put(so[i].rows, D.rows, D.nrows * 4));
    CUDA_TRY(put(so[i].lp, S.level_ptr.data(), S.level_ptr.size() * 4));
    CUDA_TRY(put(so[i].st, S.chain_recs.data(), S.chain_recs.size() * 4));
    S.d_rp = (const int32_t*)(A + so[i].rp);
    S.d_ci = (const int32_t*)(A + so[i].ci);
    S.d_val = (const void*)(A + so[i].val);
    S.d_rows = (const int32_t*)(A + so[i].rows);
    S.d_level_ptr = (const int32_t*)(A + so[i].lp);
    S.d_chain_recs = (const int32_t*)(A + so[i].st);
    CUDA_TRY(put(so[i].er, S.ell_recs.data(), S.ell_recs.size() * 4));
    CUDA_TRY(put(so[i].ed, S.ell_data.data(), S.ell_data.size()));
    S.d_ell_recs = (const int32_t*)(A + so[i].er);
    S.d_ell_data = (const char*)(A + so[i].ed);
    CUDA_TRY(put(so[i].sd, S.sn_desc.data(), S.sn_desc.size()));
    CUDA_TRY(put(so[i].sc, S.sn_cols.data(), S.sn_cols.size() * 4));
    CUDA_TRY(put(so[i].sv, S.sn_vals.data(), S.sn_vals.size()));
    CUDA_TRY(put(so[i].sbk, S.sn_blk.data(), S.sn_blk.size()));
    S.d_sn_desc = (const void*)(A + so[i].sd);
    S.d_sn_cols = (const int32_t*)(A + so[i].sc);
    S.d_sn_vals = (const void*)(A + so[i].sv);
    S.d_sn_blk = (const void*)(A + so[i].sbk);
    CUDA_TRY(put(so[i].ps, S.wave_strands.data(), S.wave_strands.size()));
    CUDA_TRY(put(so[i].pd, S.wave_data.data(), S.wave_data.size()));
    S.d_wave_strands = (const void*)(A + so[i].ps);
    S.d_wave_data = (const char*)(A + so[i].pd);
    CUDA_TRY(put(so[i].pc, S.wave_crows.data(), S.wave_crows.size() * 4));
    S.d_wave_crows = (const int32_t*)(A + so[i].pc);
    CUDA_TRY(put(so[i].sq, S.sq_items.data(), S.sq_items.size() * 4));
    S.d_sq_items = (const int32_t*)(A + so[i].sq);
    CUDA_TRY(put(so[i].sf, S.sf_items.data(), S.sf_items.size() * 4));
    S.d_sf_items = (const int32_t*)(A + so[i].sf);
    CUDA_TRY(put(so[i].sni, S.sn_items.data(), S.sn_items.size() * 4));
    S.d_sn_items = (const int32_t*)(A + so[i].sni);
  }
  if (std::getenv("SPTRSV_TEST_WEDGE")) {
    // test hook (DEADLOCK path): the first off-diagonal entry of the first
    // sync-free triangle points at its own row, which then never becomes ready
    for (size_t i = 0; i < p.segs.size(); ++i) {
      Segment& S = p.segs[i];
      if (S.info.kind != 0 || S.info.impl != SPTRSV_IMPL_TRI_SYNCFREE || S.ci.empty()) continue;
      const int m = S.info.row1 - S.info.row0;
      for (int r = 0; r < m; ++r)
        if (S.rp[r + 1] > S.rp[r]) {
          const int32_t self = S.info.row0 + r;
          CUDA_TRY(cudaMemcpyAsync(A + so[i].ci + (size_t)S.rp[r] * 4, &self, 4, cudaMemcpyHostToDevice, s));
          CUDA_TRY(cudaStreamSynchronize(s));
          break;
        }
      break;
    }
  }
  p.d_perm = (const int32_t*)(A + o_perm);
  p.d_rdiag = (const void*)(A + o_rdiag);
  p.d_tickets = (uint32_t*)(A + o_tickets);
  p.d_derr = (int32_t*)(A + o_ctl);
  p.d_epoch = (uint32_t*)(A + o_ctl + 8);
  p.d_part = (void*)(A + o_part);
  clk.lap("upload: H2D copies issued");
  // mapped host word for the spin-wait watchdog, from a process-wide pool
  // (cudaHostAlloc costs milliseconds per call)
  if (!watchdog_word_acquire(&p.h_error, &p.d_error)) {
    p.h_error = nullptr;
    p.d_error = nullptr;
  } else {
    *p.h_error = 0;
  }
  if (p.opts.max_nrhs > 0) {  // size the solve workspace now (no allocation at solve time)
    Error e = prepare_solve(p, p.opts.max_nrhs, s);
    if (e.status) return e;
    p.epoch = 0;  // prepare_solve counted a solve that did not happen
  }
  CUDA_TRY(cudaStreamSynchronize(s));
  clk.lap("upload: H2D complete");
  p.launches_per_solve = count_launches(p);
  return {SPTRSV_SUCCESS, ""};
}

// End-to-end solve from HOST buffers with many column-major right-hand
// sides: the columns are cut into blocks of cb; block k's host->device copy
// (stream h2d), its solve (the caller's stream) and its device->host copy
// (stream d2h) overlap the neighbouring blocks', over two staging buffers
// per direction.  PCIe runs both directions at once, so the call costs about
// one direction's transfer instead of transfer-in + solve + transfer-out.
Error solve_host_pipelined(Plan& p, const void* b, int64_t ldb, void* x, int64_t ldx, int32_t nrhs,
                           cudaStream_t s) {
  const size_t vb = p.vbytes;
  const int nblk = std::min(8, std::max(2, nrhs / 16));
  const int cb = (nrhs + nblk - 1) / nblk;
  const size_t blk_bytes = (size_t)p.n * cb * vb;
  if (2 * blk_bytes > p.ws.stage_bytes) {
    CUDA_TRY(cudaStreamSynchronize(s));  // the old staging may still be in use
    dfree(p, p.ws.stage_b, s);
    dfree(p, p.ws.stage_x, s);
    p.ws.stage_b = p.ws.stage_x = nullptr;
    p.ws.stage_bytes = 0;
    p.ws.stage_b = dalloc(p, 2 * blk_bytes, s);
    p.ws.stage_x = dalloc(p, 2 * blk_bytes, s);
    if (!p.ws.stage_b || !p.ws.stage_x) return {SPTRSV_ERROR_ALLOC, "staging allocation failed"};
    p.ws.stage_bytes = 2 * blk_bytes;
  }
  if (!p.ws.h2d) {
    cudaStream_t a, c;
    CUDA_TRY(cudaStreamCreateWithFlags(&a, cudaStreamNonBlocking));
    CUDA_TRY(cudaStreamCreateWithFlags(&c, cudaStreamNonBlocking));
    p.ws.h2d = (void*)a;
    p.ws.d2h = (void*)c;
    for (auto& e : p.ws.ev) {
      cudaEvent_t ev;
      CUDA_TRY(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
      e = (void*)ev;
    }
  }
  cudaStream_t h2d = (cudaStream_t)p.ws.h2d, d2h = (cudaStream_t)p.ws.d2h;
  cudaEvent_t* ev = (cudaEvent_t*)p.ws.ev;  // in[0..1], comp[2..3], out[4..5]
  // the copy streams start after whatever the caller queued on s
  CUDA_TRY(cudaEventRecord(ev[2], s));
  CUDA_TRY(cudaEventRecord(ev[3], s));
  CUDA_TRY(cudaEventRecord(ev[4], s));
  CUDA_TRY(cudaEventRecord(ev[5], s));
  const size_t width = (size_t)p.n * vb;
  for (int k = 0; k * cb < nrhs; ++k) {
    const int c0 = k * cb, nc = std::min(cb, nrhs - c0), u = k & 1;
    char* sb = (char*)p.ws.stage_b + u * blk_bytes;
    char* sx = (char*)p.ws.stage_x + u * blk_bytes;
    // in: stage_b[u] is free once the solve of block k-2 finished
    CUDA_TRY(cudaStreamWaitEvent(h2d, ev[2 + u], 0));
    CUDA_TRY(cudaMemcpy2DAsync(sb, width, (const char*)b + (size_t)c0 * ldb * vb, (size_t)ldb * vb, width, nc,
                               cudaMemcpyHostToDevice, h2d));
    CUDA_TRY(cudaEventRecord(ev[u], h2d));
    // solve: needs block k in, and stage_x[u] drained by block k-2's copy out
    CUDA_TRY(cudaStreamWaitEvent(s, ev[u], 0));
    CUDA_TRY(cudaStreamWaitEvent(s, ev[4 + u], 0));
    Error e = solve_device_any(p, sb, p.n, sx, p.n, nc, SPTRSV_COL_MAJOR, s);
    if (e.status) return e;
    CUDA_TRY(cudaEventRecord(ev[2 + u], s));
    // out
    CUDA_TRY(cudaStreamWaitEvent(d2h, ev[2 + u], 0));
    CUDA_TRY(cudaMemcpy2DAsync((char*)x + (size_t)c0 * ldx * vb, (size_t)ldx * vb, sx, width, width, nc,
                               cudaMemcpyDeviceToHost, d2h));
    CUDA_TRY(cudaEventRecord(ev[4 + u], d2h));
  }
  CUDA_TRY(cudaStreamSynchronize(d2h));
  CUDA_TRY(cudaStreamSynchronize(s));
  return {SPTRSV_SUCCESS, ""};
}

// A trip of the spin-wait watchdog during an earlier solve: report it once
// and re-arm (host mapped word and its device copy).
bool take_deadlock(Plan& p, cudaStream_t s) {
  if (!(p.h_error && *(volatile int32_t*)p.h_error)) return false;
  *(volatile int32_t*)p.h_error = 0;
  if (p.d_derr) cudaMemsetAsync(p.d_derr, 0, 4, s);
  return true;
}

Error record_done(Plan& p, cudaStream_t s) {
  if (!p.done_ev) {
    cudaEvent_t e;
    CUDA_TRY(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    p.done_ev = (void*)e;
  }
  CUDA_TRY(cudaEventRecord((cudaEvent_t)p.done_ev, s));
  p.done_ev_recorded = true;
  return {SPTRSV_SUCCESS, ""};
}

// Device solve with CUDA-graph reuse (opts.graphs): a key (b, x, ld, nrhs,
// layout) seen twice in a row is captured -- on the plan's private capture
// stream, so the caller's stream may be the legacy default stream -- and
// every later solve with a captured key is one cudaGraphLaunch.
Error solve_device_graphed(Plan& p, const void* b, int64_t ldb, void* x, int64_t ldx, int32_t nrhs,
                           sptrsv_layout_t layout, cudaStream_t s) {
  Error e = prepare_solve(p, nrhs, s);
  if (e.status) return e;
  auto eager = [&]() {
    return p.dtype == SPTRSV_R64F
               ? solve_device<double>(p, (const double*)b, ldb, (double*)x, ldx, nrhs, layout, s)
               : solve_device<float>(p, (const float*)b, ldb, (float*)x, ldx, nrhs, layout, s);
  };
  bool use_graph = p.opts.graphs != 0 && !p.profiling && !p.trace && !p.d_sf_trace;
  if (use_graph) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    CUDA_TRY(cudaStreamIsCapturing(s, &cs));
    if (cs != cudaStreamCaptureStatusNone) use_graph = false;  // inside the caller's own capture
  }
  if (!use_graph) return eager();
  ++p.solve_count;
  auto same = [&](const GraphEntry& g) {
    return g.b == b && g.x == x && g.ldb == ldb && g.ldx == ldx && g.nrhs == nrhs && g.layout == (int)layout;
  };
  for (auto& g : p.graphs)
    if (same(g)) {
      g.last_use = p.solve_count;
      CUDA_TRY(cudaGraphLaunch((cudaGraphExec_t)g.exec, s));
      return {SPTRSV_SUCCESS, ""};
    }
  if (!same(p.pending)) {  // first sighting: run eagerly, remember the key
    p.pending = GraphEntry{b, x, ldb, ldx, nrhs, (int)layout, nullptr, 0};
    return eager();
  }
  // second sighting in a row: capture
  if (!p.capture_stream) {
    cudaStream_t c;
    CUDA_TRY(cudaStreamCreateWithFlags(&c, cudaStreamNonBlocking));
    p.capture_stream = (void*)c;
  }
  cudaStream_t cs = (cudaStream_t)p.capture_stream;
  CUDA_TRY(cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal));
  Error ce = p.dtype == SPTRSV_R64F
                 ? solve_device<double>(p, (const double*)b, ldb, (double*)x, ldx, nrhs, layout, cs)
                 : solve_device<float>(p, (const float*)b, ldb, (float*)x, ldx, nrhs, layout, cs);
  cudaGraph_t graph = nullptr;
  cudaError_t ee = cudaStreamEndCapture(cs, &graph);
  if (ce.status || ee != cudaSuccess || !graph) {
    if (graph) cudaGraphDestroy(graph);
    cudaGetLastError();
    p.pending = GraphEntry{};
    if (ce.status) return ce;
    return eager();  // capture not possible here: plain launches
  }
  cudaGraphExec_t exec = nullptr;
  ee = cudaGraphInstantiate(&exec, graph, 0);
  cudaGraphDestroy(graph);
  if (ee != cudaSuccess) {
    cudaGetLastError();
    p.pending = GraphEntry{};
    return eager();
  }
  if (p.graphs.size() >= 8) {  // evict the least recently used
    auto lru = std::min_element(p.graphs.begin(), p.graphs.end(),
                                [](const GraphEntry& a2, const GraphEntry& b2) { return a2.last_use < b2.last_use; });
    cudaGraphExecDestroy((cudaGraphExec_t)lru->exec);
    p.graphs.erase(lru);
  }
  GraphEntry g = p.pending;
  g.exec = (void*)exec;
  g.last_use = p.solve_count;
  p.graphs.push_back(g);
  p.pending = GraphEntry{};
  CUDA_TRY(cudaGraphLaunch(exec, s));
  return {SPTRSV_SUCCESS, ""};
}

Error solve(Plan& p, const void* b, int64_t ldb, void* x, int64_t ldx, int32_t nrhs, sptrsv_layout_t layout,
            void* stream_v) {
  cudaStream_t s = (cudaStream_t)stream_v;
  // the plan is bound to its device (our runtime's current device is not
  // torch's: make it explicit on every call)
  int cur = -1;
  if (cudaGetDevice(&cur) != cudaSuccess || cur != p.device) CUDA_TRY(cudaSetDevice(p.device));
  if (take_deadlock(p, s))
    return {SPTRSV_ERROR_DEADLOCK, "a spin-wait watchdog tripped during an earlier solve on this plan"};
  if (nrhs == 0 || p.n == 0) return {SPTRSV_SUCCESS, ""};
  int bdev = -1, xdev = -1;
  const int bd = ptr_kind(b, &bdev), xd = ptr_kind(x, &xdev);
  if (bd != xd) return {SPTRSV_ERROR_INVALID_VALUE, "b and x must both be device or both be host pointers"};
  const size_t vb = p.vbytes;
  if (bd) {
    if (bdev != p.device || xdev != p.device)
      return {SPTRSV_ERROR_INVALID_VALUE, "b / x live on device " + std::to_string(bdev) + " / " +
                                              std::to_string(xdev) + ", the plan on device " +
                                              std::to_string(p.device)};
    Error e = solve_device_graphed(p, b, ldb, x, ldx, nrhs, layout, s);
    if (e.status) return e;
    return record_done(p, s);
  }
  Error out{SPTRSV_SUCCESS, ""};
  // host buffers, many column-major RHS: pipelined by column blocks
  if (layout == SPTRSV_COL_MAJOR && nrhs >= 32 && std::getenv("SPTRSV_NO_PIPELINE") == nullptr) {
    out = solve_host_pipelined(p, b, ldb, x, ldx, nrhs, s);
  } else {
    // host buffers: stage through the device (end-to-end path), then sync
    size_t need = (size_t)p.n * nrhs * vb;
    if (need > p.ws.stage_bytes) {
      CUDA_TRY(cudaStreamSynchronize(s));
      dfree(p, p.ws.stage_b, s);
      dfree(p, p.ws.stage_x, s);
      p.ws.stage_b = p.ws.stage_x = nullptr;
      p.ws.stage_bytes = 0;
      p.ws.stage_b = dalloc(p, need, s);
      p.ws.stage_x = dalloc(p, need, s);
      if (!p.ws.stage_b || !p.ws.stage_x) return {SPTRSV_ERROR_ALLOC, "staging allocation failed"};
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
    Error e = solve_device_any(p, p.ws.stage_b, dld, p.ws.stage_x, dld, nrhs, layout, s);
    if (e.status) return e;
    CUDA_TRY(cudaMemcpy2DAsync(x, (size_t)ldx * vb, p.ws.stage_x, width, width, height, cudaMemcpyDeviceToHost, s));
    CUDA_TRY(cudaStreamSynchronize(s));
  }
  if (out.status) return out;
  Error e = record_done(p, s);
  if (e.status) return e;
  if (take_deadlock(p, s)) return {SPTRSV_ERROR_DEADLOCK, "spin-wait watchdog tripped"};
  return {SPTRSV_SUCCESS, ""};
}

// ------------------------------------------- A^T x = b from the same plan
// (reading R32; kernels: k::perm_in_T / tri_push_T /
// sq_push_T / perm_out_T).  First call: the in-degree counters of L1^T
// (column counts of every triangle's CSR) and, for wave triangles whose
// device row order is not the level order, the reverse-level claim order.
Error prepare_T(Plan& p, cudaStream_t s) {
  if (p.d_tcnt0) return {SPTRSV_SUCCESS, ""};
  const int n = p.n;
  const size_t ns = p.segs.size();
  p.d_tcnt0 = (int32_t*)dalloc(p, (size_t)std::max(1, n) * 4, s);
  p.d_tcnt = (int32_t*)dalloc(p, (size_t)std::max(1, n) * 4, s);
  p.d_tticket = (uint32_t*)dalloc(p, std::max<size_t>(1, ns) * 4, s);
  if (!p.d_tcnt0 || !p.d_tcnt || !p.d_tticket) return {SPTRSV_ERROR_ALLOC, "transposed-solve workspace"};
  CUDA_TRY(cudaMemsetAsync(p.d_tcnt0, 0, (size_t)std::max(1, n) * 4, s));
  p.d_torder.assign(ns, nullptr);
  p.d_tpos.assign(ns, nullptr);
  p.d_tlvs.assign(ns, nullptr);
  p.d_ttpos.assign(ns, nullptr);
  p.d_tpc.assign(ns, PcSeg{});
  auto upload_ints = [&](const std::vector<int32_t>& h, int32_t** d) -> Error {
    *d = (int32_t*)dalloc(p, std::max<size_t>(1, h.size()) * 4, s);
    if (!*d) return {SPTRSV_ERROR_ALLOC, "transposed-solve index arrays"};
    CUDA_TRY(cudaMemcpyAsync(*d, h.data(), h.size() * 4, cudaMemcpyHostToDevice, s));
    CUDA_TRY(cudaStreamSynchronize(s));  // h is a host temporary
    return {SPTRSV_SUCCESS, ""};
  };
  for (size_t i = 0; i < ns; ++i) {
    Segment& S = p.segs[i];
    if (S.info.kind != 0) continue;
    const int m = S.info.row1 - S.info.row0;
    const int64_t ne = S.rp.empty() ? (int64_t)S.info.nnz - m : (int64_t)S.rp.back();
    if (ne > 0)
      k::count_cols<<<(unsigned)std::min<int64_t>(cdiv(ne, 256), (int64_t)p.sm_count * 16), 256, 0, s>>>(
          ne, S.d_ci, p.d_tcnt0);
    const bool wave = S.wave_K > 0 && (int)S.wave_tau.size() == m;
    std::vector<int32_t> ord;
    if (wave) {  // device position q of plan row t: tau^-1
      std::vector<int32_t> inv(m), pos(m);
      ord.resize(m);
      for (int q = 0; q < m; ++q) inv[S.wave_tau[q]] = q;
      for (int i2 = 0; i2 < m; ++i2) ord[i2] = inv[m - 1 - i2];
      for (int q = 0; q < m; ++q) pos[q] = m - 1 - S.wave_tau[q];
      Error e = upload_ints(ord, &p.d_torder[i]);
      if (e.status) return e;
      e = upload_ints(pos, &p.d_tpos[i]);
      if (e.status) return e;
    }
    // narrow-level triangle (levels contiguous in plan order, every level <=
    // kPcMaxW rows, enough levels to be latency-bound): one-CTA reverse chain
    const int nl = S.info.nlevels;
    if (p.reorder_eff == 0 && nl >= 32 && (int)S.level_ptr.size() == nl + 1 &&
        std::getenv("SPTRSV_NO_PUSHCHAIN") == nullptr) {
      int wmax = 0;
      for (int l = 0; l < nl; ++l) wmax = std::max(wmax, S.level_ptr[l + 1] - S.level_ptr[l]);
      if (wmax <= k::kPcMaxW) {
        std::vector<int32_t> lvs(nl + 1);
        for (int l = 0; l <= nl; ++l) lvs[l] = m - S.level_ptr[nl - l];
        Error e = upload_ints(lvs, &p.d_tlvs[i]);
        if (e.status) return e;
        p.d_ttpos[i] = (int32_t*)dalloc(p, (size_t)std::max<int64_t>(1, ne) * 4, s);
        if (!p.d_ttpos[i]) return {SPTRSV_ERROR_ALLOC, "transposed-solve target positions"};
        if (ne > 0)
          k::pc_tpos<<<(unsigned)std::min<int64_t>(cdiv(ne, 256), (int64_t)p.sm_count * 16), 256, 0, s>>>(
              ne, S.info.row0, m, S.d_ci, p.d_tpos[i], p.d_ttpos[i]);
        // claim-position records: row, entry count, first kPcE (target, value) pairs; b' buffer
        std::vector<int32_t> pq(m);
        for (int q2 = 0; q2 < m; ++q2) pq[q2] = wave ? ord[q2] : m - 1 - q2;
        PcSeg& C = p.d_tpc[i];
        e = upload_ints(pq, &C.pq);
        if (e.status) return e;
        C.ecnt = (int32_t*)dalloc(p, (size_t)m * 4, s);
        C.etp = (int32_t*)dalloc(p, (size_t)m * k::kPcE * 4, s);
        C.ev = dalloc(p, (size_t)m * k::kPcE * p.vbytes, s);
        C.gpos = dalloc(p, (size_t)m * p.vbytes, s);
        if (!C.ecnt || !C.etp || !C.ev || !C.gpos) return {SPTRSV_ERROR_ALLOC, "transposed-solve chain records"};
        if (p.vbytes == 8)
          k::pc_build<double><<<cdiv(m, 256), 256, 0, s>>>(m, C.pq, S.d_rp, p.d_ttpos[i], (const double*)S.d_val,
                                                           C.ecnt, C.etp, (double*)C.ev);
        else
          k::pc_build<float><<<cdiv(m, 256), 256, 0, s>>>(m, C.pq, S.d_rp, p.d_ttpos[i], (const float*)S.d_val,
                                                          C.ecnt, C.etp, (float*)C.ev);
        CUDA_TRY(cudaGetLastError());
      }
    }
  }
  CUDA_TRY(cudaGetLastError());
  return {SPTRSV_SUCCESS, ""};
}

template <typename T>
Error solve_T_device(Plan& p, const T* b, int64_t ldb, T* x, int64_t ldx, sptrsv_layout_t layout, cudaStream_t s) {
  const int n = p.n;
  T* bw = (T*)p.ws.bw;
  T* xs = (T*)p.ws.xs;
  k::SolveState st{p.d_tickets, p.nticket, p.d_error, nullptr, p.d_epoch, 0u, 0u, p.backoff_ns, p.d_derr, p.wd_spins,
                   nullptr};
  const int64_t sb = layout == SPTRSV_ROW_MAJOR ? ldb : 1, sx = layout == SPTRSV_ROW_MAJOR ? ldx : 1;
  const int nseg = (int)p.segs.size();
  k::perm_in_T<T><<<std::max(1u, cdiv(n, 256)), 256, 0, s>>>(n, p.d_perm, b, sb, bw, p.d_tcnt0, p.d_tcnt,
                                                             p.d_tticket, nseg);
  CUDA_TRY(cudaGetLastError());
  for (int si = nseg - 1; si >= 0; --si) {  // segments in reverse order
    Segment& S = p.segs[si];
    const auto& I = S.info;
    const T* val = (const T*)S.d_val;
    if (I.kind == 1) {
      if (S.dev_nzr > 0 && I.nnz > 0) {
        const unsigned g = cdiv(S.dev_nzr, 128);
        if (S.dev_dcsr)
          k::sq_push_T<T, true><<<g, 128, 0, s>>>(S.dev_nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs, bw);
        else
          k::sq_push_T<T, false><<<g, 128, 0, s>>>(S.dev_nzr, I.row0, S.d_rows, S.d_rp, S.d_ci, val, xs, bw);
      }
    } else {
      const int m = I.row1 - I.row0;
      if (m > 0 && p.d_tlvs[si]) {  // narrow levels: one-CTA reverse chain, shared-memory ring
        constexpr int XW = 2 * k::kPcMaxW * 2;  // >= 2 levels of kPcMaxW rows, a power of two
        const uint32_t smem = (uint32_t)(XW * sizeof(T));
        auto kern = k::tri_pushchain_T<T>;
        CUDA_TRY(ensure_smem_attr((const void*)kern, smem, false));
        const PcSeg& C = p.d_tpc[si];
        k::pc_gather<T><<<cdiv(m, 256), 256, 0, s>>>(m, I.row0, C.pq, bw, (T*)C.gpos);
        kern<<<1, k::kPcNT, smem, s>>>(I.row0, I.nlevels, p.d_tlvs[si], C.pq, C.ecnt, C.etp, (const T*)C.ev,
                                       (T*)C.gpos, S.d_rp, p.d_ttpos[si], val, xs, XW);
      } else if (m > 0) {
        const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>(cdiv(m, 256), (int64_t)p.sm_count * 2));
        k::tri_push_T<T><<<g, 256, 0, s>>>(I.row0, m, p.d_torder.empty() ? nullptr : p.d_torder[si], S.d_rp, S.d_ci,
                                           val, bw, xs, p.d_tcnt, p.d_tticket + si, st);
      }
    }
    CUDA_TRY(cudaGetLastError());
  }
  k::perm_out_T<T><<<std::max(1u, cdiv(n, 256)), 256, 0, s>>>(n, p.d_perm, (const T*)p.d_rdiag, xs, x, sx);
  CUDA_TRY(cudaGetLastError());
  return {SPTRSV_SUCCESS, ""};
}

Error solve_T(Plan& p, const void* b, int64_t ldb, void* x, int64_t ldx, int32_t nrhs, sptrsv_layout_t layout,
              void* stream_v) {
  cudaStream_t s = (cudaStream_t)stream_v;
  int cur = -1;
  if (cudaGetDevice(&cur) != cudaSuccess || cur != p.device) CUDA_TRY(cudaSetDevice(p.device));
  if (take_deadlock(p, s))
    return {SPTRSV_ERROR_DEADLOCK, "a spin-wait watchdog tripped during an earlier solve on this plan"};
  if (nrhs == 0 || p.n == 0) return {SPTRSV_SUCCESS, ""};
  if (nrhs != 1) return {SPTRSV_ERROR_NOT_SUPPORTED, "the transposed solve from the same plan takes one RHS"};
  int bdev = -1, xdev = -1;
  const int bd = ptr_kind(b, &bdev), xd = ptr_kind(x, &xdev);
  if (!bd || !xd) return {SPTRSV_ERROR_NOT_SUPPORTED, "the transposed solve takes device pointers"};
  if (bdev != p.device || xdev != p.device)
    return {SPTRSV_ERROR_INVALID_VALUE, "b / x live on another device than the plan"};
  Error e = prepare_solve(p, 1, s);
  if (e.status) return e;
  e = prepare_T(p, s);
  if (e.status) return e;
  e = p.dtype == SPTRSV_R64F ? solve_T_device<double>(p, (const double*)b, ldb, (double*)x, ldx, layout, s)
                             : solve_T_device<float>(p, (const float*)b, ldb, (float*)x, ldx, layout, s);
  if (e.status) return e;
  return record_done(p, s);
}

void release(Plan& p) {
  if (p.device >= 0) {
    cudaSetDevice(p.device);
    // wait for this plan's last solve only (not the whole device)
    if (p.done_ev && p.done_ev_recorded) cudaEventSynchronize((cudaEvent_t)p.done_ev);
  }
  drop_graphs(p);
  if (p.capture_stream) cudaStreamDestroy((cudaStream_t)p.capture_stream);
  if (p.done_ev) cudaEventDestroy((cudaEvent_t)p.done_ev);
  dfree(p, p.arena, nullptr);
  dfree(p, p.ws.bw, nullptr);
  dfree(p, p.ws.xs, nullptr);
  dfree(p, p.ws.stage_b, nullptr);
  dfree(p, p.ws.stage_x, nullptr);
  dfree(p, p.ws.flags, nullptr);
  dfree(p, p.d_tcnt0, nullptr);
  dfree(p, p.d_tcnt, nullptr);
  dfree(p, p.d_tticket, nullptr);
  for (auto* q : p.d_torder) dfree(p, q, nullptr);
  for (auto* q : p.d_tpos) dfree(p, q, nullptr);
  for (auto* q : p.d_tlvs) dfree(p, q, nullptr);
  for (auto* q : p.d_ttpos) dfree(p, q, nullptr);
  for (auto& C : p.d_tpc) {
    dfree(p, C.pq, nullptr);
    dfree(p, C.ecnt, nullptr);
    dfree(p, C.etp, nullptr);
    dfree(p, C.ev, nullptr);
    dfree(p, C.gpos, nullptr);
  }
  p.d_tpc.clear();
  p.d_ttpos.clear();
  p.d_tpos.clear();
  p.d_tlvs.clear();
  p.d_tcnt0 = p.d_tcnt = nullptr;
  p.d_tticket = nullptr;
  p.d_torder.clear();
  if (p.ws.h2d) cudaStreamDestroy((cudaStream_t)p.ws.h2d);
  if (p.ws.d2h) cudaStreamDestroy((cudaStream_t)p.ws.d2h);
  for (void* e : p.ws.ev)
    if (e) cudaEventDestroy((cudaEvent_t)e);
  if (p.h_error) watchdog_word_release(p.h_error);
  for (auto& S : p.segs)
    if (S.d_trace) cudaFree(S.d_trace);
  if (p.d_sf_trace) cudaFree(p.d_sf_trace);
  p.d_sf_trace = nullptr;
  for (void* e : p.events) cudaEventDestroy((cudaEvent_t)e);
  p.arena = nullptr;
  p.ws = Workspace{};
  p.h_error = nullptr;
  p.events.clear();
  p.capture_stream = nullptr;
  p.done_ev = nullptr;
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
  // attribute queries (cudaGetDeviceProperties costs milliseconds per call)
  CUDA_TRY(cudaDeviceGetAttribute(sm_count, cudaDevAttrMultiProcessorCount, dev));
  CUDA_TRY(cudaDeviceGetAttribute(major, cudaDevAttrComputeCapabilityMajor, dev));
  CUDA_TRY(cudaDeviceGetAttribute(minor, cudaDevAttrComputeCapabilityMinor, dev));
  return {SPTRSV_SUCCESS, ""};
}

int count_launches_public(const Plan& p) { return count_launches(p); }
SpmmCfg spmm_cfg_public() { return spmm_cfg(); }
Error prepare_solve_public(Plan& p, int nrhs, cudaStream_t s) { return prepare_solve(p, nrhs, s); }

}  // namespace sptrsv
