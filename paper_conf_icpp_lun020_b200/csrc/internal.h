// Internal plan representation of the B200 recursive-block SpTRSV library.
// Not part of the ABI; see include/sptrsv.h.
#pragma once

#include <algorithm>
#include <chrono>
#include <cstdint>
#include <functional>
#include <thread>
#include <cstdio>
#include <cstdlib>
#include <memory>
#include <string>
#include <vector>

#include <cuda_runtime.h>

#include "sptrsv.h"

namespace sptrsv {

// Status carrier used inside the library (never crosses the ABI as C++).
struct Error {
  sptrsv_status_t status;
  std::string msg;
};

void set_last_error(const std::string& msg);

// Allocator whose resize() leaves new elements default-initialised (i.e.
// unwritten for scalars): the big index/value arrays of the analysis are
// then first touched by the threads that fill them, in parallel, instead of
// being zero-filled serially by resize().
template <class T>
struct DefaultInit : std::allocator<T> {
  template <class U>
  struct rebind { using other = DefaultInit<U>; };
  DefaultInit() = default;
  template <class U>
  DefaultInit(const DefaultInit<U>&) noexcept {}
  template <class U>
  void construct(U* p) noexcept { ::new ((void*)p) U; }
  template <class U, class... A>
  void construct(U* p, A&&... a) { ::new ((void*)p) U(std::forward<A>(a)...); }
};
template <class T>
using dvec = std::vector<T, DefaultInit<T>>;

// Run f(lo, hi) over [0, n) split into contiguous chunks on `threads`
// threads (threads <= 0: hardware concurrency, capped at 64); small ranges
// run inline.
inline void par_for(int64_t n, int threads, const std::function<void(int64_t, int64_t)>& f,
                    int64_t grain = 65536) {
  if (threads <= 0) threads = (int)std::min(64u, std::max(1u, std::thread::hardware_concurrency()));
  if (threads <= 1 || n < grain) {
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

// Phase stopwatch of the preprocessing (SPTRSV_ANALYSE_TRACE=1 prints every
// lap to stderr); costs one clock read per phase otherwise.
struct PhaseClock {
  bool on = std::getenv("SPTRSV_ANALYSE_TRACE") != nullptr;
  std::chrono::steady_clock::time_point t = std::chrono::steady_clock::now();
  void lap(const char* what) {
    if (!on) return;
    auto now = std::chrono::steady_clock::now();
    std::fprintf(stderr, "[sptrsv analyse] %-28s %9.2f ms\n", what,
                 std::chrono::duration<double, std::milli>(now - t).count());
    t = now;
  }
};

// One block of the reordered matrix P L P^T in execution order (Fig. 3(d),
// PAPER.md:L229/L235): a triangle (solved) or a rectangle (b -= A x).
struct Segment {
  sptrsv_seg_info_t info{};
  // ----- host copies (introspection + upload) -----
  // TRI: off-diagonal entries only (the diagonal lives in Plan::diag_new).
  // SQ : entries inside rows [row0,row1) x cols [col0,col1).
  // CSR rows are local (0..m-1 for CSR, 0..nzr-1 for DCSR); columns are GLOBAL
  // permuted indices so kernels index the permuted vector directly.
  std::vector<int32_t> rp;         // CSR/DCSR row pointer (local offsets)
  dvec<int32_t> ci;                // global permuted column index
  dvec<char> val;                  // dtype values
  std::vector<int32_t> rows;       // DCSR: global permuted row of every stored row
  std::vector<int32_t> level_ptr;  // TRI: nlevels+1 local row offsets
  std::vector<int32_t> in_degree;  // TRI: off-diagonal count per local row
  std::vector<int32_t> sn_ptr;     // TRI: fundamental-supernode pieces (<= 32 rows), local row starts + m
  int32_t nzr = 0;                 // SQ: stored rows (== m for CSR)
  int32_t kmax_indeg = 0;          // TRI: largest in_degree (selector feature)
  int64_t npieces = 0;             // TRI: fundamental-supernode pieces (selector feature)
  // ----- device -----
  const int32_t* d_rp = nullptr;
  const int32_t* d_ci = nullptr;
  const void* d_val = nullptr;
  const int32_t* d_rows = nullptr;
  const int32_t* d_level_ptr = nullptr;  // device copy (chain / level-set kernels)
  int32_t ticket_slot = -1;              // sync-free: index into the device ticket array
  // supernodal kernel (nrhs == 1): piece descriptors, shared external
  // column lists, dense external values (column-major, ld = width) and the
  // packed strictly-lower diagonal blocks
  std::vector<char> sn_desc;
  dvec<char> sn_vals, sn_blk;
  std::vector<int32_t> sn_cols;
  const void* d_sn_desc = nullptr;
  const int32_t* d_sn_cols = nullptr;
  const void* d_sn_vals = nullptr;
  const void* d_sn_blk = nullptr;
  std::vector<int32_t> sn_items;   // k::SnItem[] as 8 ints (pieces, or chunks of long pieces)
  const int32_t* d_sn_items = nullptr;
  int32_t sn_part_base = 0;        // first scalar of the segment's 32-wide partial slots in `part`
  // strand wavefront over a cluster (k::tri_wave, nrhs == 1); wave_K == 0: not built
  int wave_K = 0, wave_E = 0, wave_C = 0, wave_W = 0, wave_GPC = 0, wave_NCH = 0, wave_XW = 0, wave_xa = 0;
  uint32_t wave_chunk_bytes = 0, wave_bring_bytes = 0, wave_group_bytes = 0;
  int wave_ipl = 0;                // words per lane of a chunk's first-use import list
  int64_t wave_global = 0;         // dependencies polled in global memory (needs the xs sentinel)
  std::vector<int32_t> wave_tau;   // execution position q -> local row (the device row order of the triangle)
  std::vector<char> wave_strands;  // k::WaveStrand[C * W]
  std::vector<char> wave_data;     // chunk blocks
  std::vector<int32_t> wave_crows; // {lo, hi} b' rows of every chunk (the producer warp's TMA windows)
  const int32_t* d_wave_crows = nullptr;
  const void* d_wave_strands = nullptr;
  const char* d_wave_data = nullptr;
  // device-side square format: a CSR square whose rows are reordered by a
  // wave triangle is uploaded as DCSR with explicit (execution-order) rows
  bool dev_dcsr = false;
  int32_t dev_nzr = 0;
  // row-block sync-free triangle kernel (k::tri_sf_items, nrhs == 1): k::SfItem[] as 8 ints
  std::vector<int32_t> sf_items;
  bool sf_mixed = false;
  int32_t fused_sq = -1;  // TRI (mixed sync-free): index of the square fused as trailing items
  bool fused = false;     // SQ: computed inside the preceding triangle's kernel at nrhs == 1
  bool sf_wrow = false;
  int32_t cl_size = 0;    // TRI: > 0 = level-set on one cluster of cl_size CTAs (k::tri_level_cluster);
                          // sf_items then holds the level-cut items followed by ip[nlevels + 1]
  int32_t cl_nitem = 0;
  const int32_t* d_sf_items = nullptr;
  // row-block square kernel (k::sq_adapt_1, nrhs == 1): k::SqItem[] as 4 ints
  std::vector<int32_t> sq_items;
  const int32_t* d_sq_items = nullptr;
  // TMA-staged chain kernel (nrhs == 1): 8-int stage records (k::StageRec),
  // empty = not staged
  std::vector<int32_t> chain_recs;
  const int32_t* d_chain_recs = nullptr;
  // ELL-staged chain kernel (nrhs == 1, rows with <= 4 window-resident deps)
  int ell_K = 0, ell_NST = 0, ell_RMAX = 0, ell_PMAX = 0, ell_SMAX = 0, ell_XW = 0, ell_warps = 8;  // ell_K == 0: not used
  std::vector<int32_t> ell_recs;   // 16 ints per stage (k::EllRec + the record of stage s + NST)
  std::vector<char> ell_data;      // per-stage blocks: step records int4[nsteps], u16 slot pairs [W][npad], values [K][npad]
  const int32_t* d_ell_recs = nullptr;
  const char* d_ell_data = nullptr;
  void* d_trace = nullptr;          // debug trace (SPTRSV_TRACE)
  std::vector<long long> h_trace;
};

struct Workspace {
  void* bw = nullptr;       // permuted right-hand side being updated, n x nrhs row-major
  void* xs = nullptr;       // permuted solution, n x nrhs row-major
  size_t w_bytes = 0;
  void* stage_b = nullptr;  // host-pointer path staging (col-major n x nrhs)
  void* stage_x = nullptr;
  size_t stage_bytes = 0;
  void* flags = nullptr;    // nrhs > 1 sync-free: per-row ready flags (n x u32), epoch-valued
  int flags_n = 0;
  // pipelined host path (exec.cu solve_host_pipelined): copy streams + events
  void* h2d = nullptr;      // cudaStream_t
  void* d2h = nullptr;
  void* ev[6] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};  // in[2], comp[2], out[2]
};

// A captured solve (CUDA graph) for one argument set; replayed when a later
// device solve has the same key (exec.cu solve()).
struct GraphEntry {
  const void* b = nullptr;
  void* x = nullptr;
  int64_t ldb = 0, ldx = 0;
  int32_t nrhs = 0, layout = 0;
  void* exec = nullptr;  // cudaGraphExec_t
  uint64_t last_use = 0;
};

// SpMM lane geometry for nrhs > 1 (exec.cu: dispatch_multi_un)
struct SpmmCfg {
  int rpt_max = 8, un = 2;  // measured best on C5 (round 1 sweep, profiles/r01_sweeps.md)
  int tile = 0;             // RHS tile width of the tiled SpMM (0 = untiled, the default: re-streaming
                            // the matrix per tile measured 1.6-1.75x slower on C5; SPTRSV_SPMM_TILE)
};

// claim-position records of a narrow-level triangle's transposed chain
// (k::pc_build / pc_gather / tri_pushchain_T)
struct PcSeg {
  int32_t* pq = nullptr;    // claim position -> local device row
  int32_t* ecnt = nullptr;  // entries of that row
  int32_t* etp = nullptr;   // first kPcE target positions
  void* ev = nullptr;       // their values
  void* gpos = nullptr;     // b' in claim-position order (per solve)
};

struct Plan {
  sptrsv_opts_t opts{};
  int32_t n = 0;
  int64_t nnz = 0;
  int32_t depth = 0;
  sptrsv_dtype_t dtype = SPTRSV_R64F;
  sptrsv_fill_t fill = SPTRSV_LOWER;
  int32_t sm_count = 148;
  int64_t min_block_rows = 0;
  double analyse_ms = 0.0;
  int32_t reorder_eff = 0;  // reorder actually applied (0 level, 1 none)
  int32_t depth_retuned = 0;  // 1: the B200 selector overrode the paper's depth rule (R30)
  size_t vbytes = 8;

  std::vector<Segment> segs;
  std::vector<int32_t> perm;        // new -> old (original indexing; UPPER composed with J)
  std::vector<int32_t> leaf_level;  // level of every new row inside its leaf
  std::vector<int32_t> lower_old;   // new row -> row of the (J U J for UPPER) lower input
  std::vector<char> diag_new;       // diagonal in new order (dtype)
  std::vector<char> rdiag_new;      // 1 / diagonal in new order (dtype), what kernels read
  // P L P^T kept on the host for introspection (sptrsv_plan_matrix)
  std::vector<int64_t> p_rp;
  dvec<int32_t> p_ci;
  dvec<char> p_val;

  bool dev_analysed = false;  // the analysis ran on the device (analyse_dev.cu)
  int32_t analysis_where = 0; // 0 host, 1 device, 2 device + host-built formats
  bool host_ready = true;     // host copies of the stored arrays exist (else materialize_host)
  // ----- device -----
  int device = -1;
  const int32_t* d_leaf_level = nullptr;  // device-analysed plans: leaf levels (introspection)
  void* arena = nullptr;
  size_t arena_bytes = 0;
  const int32_t* d_perm = nullptr;
  const void* d_rdiag = nullptr;  // 1/d in new order (permute-in scaling)
  uint32_t* d_tickets = nullptr;  // [nticket] sync-free row-claim counters
  void* d_part = nullptr;         // partial sums of split long rows (k::tri_sf_items), sentinel-reset per solve
  int32_t npart = 0;
  int32_t nticket = 0;
  bool needs_sentinel = false;    // nrhs == 1: a triangle polls xs (value-as-flag)
  bool needs_flags = false;       // nrhs > 1: a sync-free triangle polls per-row epoch flags
  int chain_geom[5] = {0, 0, 0, 0, 0};  // NST, RMAX, EMAX, XW, LMAX frozen at upload
  bool trace = false;                   // SPTRSV_TRACE debug stamps
  int32_t* h_error = nullptr;  // mapped pinned host word set by the watchdog
  int32_t* d_error = nullptr;  // its device alias
  Workspace ws;
  SpmmCfg spmm;
  uint32_t backoff_ns = 128;  // sync-free polling backoff cap
  uint32_t wd_spins = 0;      // watchdog: unsuccessful polls before SPTRSV_ERROR_DEADLOCK
  void* d_sf_trace = nullptr; // SPTRSV_SF_TRACE: {claim, done} timestamps per row (debug)
  uint32_t epoch = 0;  // host mirror of the device epoch counter (wrap detection only)
  uint32_t* d_epoch = nullptr;  // device words {this solve's base epoch, last epoch handed out}
  int32_t* d_derr = nullptr;    // device copy of the watchdog word
  // CUDA graphs of repeated device solves (key: b, x, ld, nrhs, layout)
  std::vector<GraphEntry> graphs;
  GraphEntry pending;           // last uncaptured key (captured when it repeats)
  uint64_t solve_count = 0;
  void* capture_stream = nullptr;  // cudaStream_t used only to capture
  void* done_ev = nullptr;         // recorded after every solve; sptrsv_free waits on it
  bool done_ev_recorded = false;
  int launches_per_solve = 0;

  // transposed solve from the same plan (f-4, reading R32; exec.cu solve_T):
  // built at the first A^T solve
  int32_t* d_tcnt0 = nullptr;        // in-degree of L1^T per row: column counts inside its triangle
  int32_t* d_tcnt = nullptr;         // working counters, reset from d_tcnt0 by permute-in
  uint32_t* d_tticket = nullptr;     // per-segment claim tickets
  std::vector<int32_t*> d_torder;    // per segment: claim order (wave triangles), else nullptr
  std::vector<int32_t*> d_tpos;      // per segment: device row -> claim position (wave triangles)
  std::vector<int32_t*> d_ttpos;     // per segment: claim position of every CSR entry's target
  std::vector<PcSeg> d_tpc;          // per segment: claim-position records (k::tri_pushchain_T)
  std::vector<int32_t*> d_tlvs;      // per segment: claim-position level starts (narrow-level
                                     // triangles solved by k::tri_pushchain_T), else nullptr

  // profiling
  bool profiling = false;
  std::vector<void*> events;  // cudaEvent_t
  int last_nseg_timed = 0;
};

// analysis (host, deterministic); fills everything but the device fields
Error analyse_host(Plan& p, int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx,
                   const void* val);

// kernel implementation choice per segment (selector / forced)
void choose_impls(Plan& p);

// segment geometry + host extraction (analyse.cpp); used by both analyses
struct SegGeo {
  int32_t kind, r0, r1, c0, c1, leaf;
};
std::vector<SegGeo> segment_geometry(int32_t n, int32_t depth, int32_t variant,
                                     const std::vector<std::pair<int32_t, int32_t>>& leaves);
Error build_segments_host(Plan& p, const std::vector<std::pair<int32_t, int32_t>>& leaves,
                          const std::vector<int32_t>& leaf_nl, int threads);
int32_t select_tri(int32_t nlevels, int32_t npr);
int64_t default_min_block_rows(const Plan& p);  // reading R2 / R33
int32_t select_sq(int32_t npr, int64_t empty, int64_t m);

// device-resident analysis (analyse_dev.cu): CSR given as
// device pointers; builds the arena on the device (no upload()).
Error analyse_device(Plan& p, int32_t n, int64_t nnz, const int32_t* d_rp, const int32_t* d_ci, const void* d_val,
                     void* stream);
// host copies of a device-analysed plan's arrays (introspection, hash)
Error materialize_host(Plan& p);
void* dalloc(Plan& p, size_t bytes, cudaStream_t s);
void dfree(Plan& p, void* q, cudaStream_t s);

// device side (exec.cu)
Error upload(Plan& p, void* stream);
Error solve(Plan& p, const void* b, int64_t ldb, void* x, int64_t ldx, int32_t nrhs,
            sptrsv_layout_t layout, void* stream);
// A^T x = b with the plan of A (nrhs == 1, device pointers)
Error solve_T(Plan& p, const void* b, int64_t ldb, void* x, int64_t ldx, int32_t nrhs,
              sptrsv_layout_t layout, void* stream);
void release(Plan& p);

}  // namespace sptrsv
