/*
 * sptrsv.h -- C ABI of the B200-native recursive-block sparse triangular
 * solve (Lu, Niu & Liu, "Efficient Block Algorithms for Parallel Sparse
 * Triangular Solve", ICPP'20; text in PAPER.md, cited as PAPER.md:L<line>).
 *
 * Operation (Sec 1): solve L x = b (or U x = b) where L (U) is a
 * sparse lower (upper) triangular matrix in CSR, b a dense right-hand side and
 * x the dense solution.  The two-phase structure follows the paper:
 *   - sptrsv_analyse = the preprocessing stage (Sec 3.3, Sec 3.4, Alg 2
 *     L77-L87, Alg 3, Table 5 "preprocessing time"): validation,
 *     level sets, level-set reordering of every triangle (L231-L233), the
 *     recursive (Alg 6) / column (Alg 4) / row (Alg 5) block partition with
 *     the depth rule of L299, per-block features and the Alg 7 kernel choice
 *     (L252-L296), and the blocked storage in execution order (L229, L235-L241).
 *   - sptrsv_solve = IMPROVED-RECURSIVE-BLOCK-ALGORITHM (Alg 7):
 *     a loop over the stored triangles (SpTRSV) and squares (SpMV, b -= A x),
 *     for nrhs >= 1 right-hand sides (SpTRSM when nrhs > 1).
 *
 * Conventions shared by every entry point:
 *   - Every function is extern "C", never throws and never aborts; it returns
 *     an sptrsv_status_t.  sptrsv_last_error() gives a thread-local detail
 *     string for the most recent failing call on the calling thread.
 *   - Indices are 0-based int32; nnz must be < 2^31.
 *   - A "stream" argument is a cudaStream_t passed as void* (NULL = the legacy
 *     default stream).  No CUDA or torch type appears in any signature.
 *   - The library is built for sm_100a (B200) only.  There is no CPU fallback:
 *     sptrsv_solve fails with SPTRSV_ERROR_NOT_SUPPORTED on any other device.
 */
#ifndef SPTRSV_H_
#define SPTRSV_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct sptrsv_plan_s* sptrsv_plan_t; /* opaque; owned by the library */

typedef enum {
  SPTRSV_SUCCESS = 0,
  SPTRSV_ERROR_INVALID_VALUE = 1, /* null pointer, n < 0, nnz != row_ptr[n], nrhs < 0, ld < n, bad enum */
  SPTRSV_ERROR_NOT_TRIANGULAR = 2, /* entry above (LOWER) / below (UPPER) the diagonal */
  SPTRSV_ERROR_UNSORTED = 3,       /* column indices not strictly increasing in a row (incl. duplicates) */
  SPTRSV_ERROR_ZERO_PIVOT = 4,     /* diagonal missing or exactly 0 (row index in sptrsv_last_error) */
  SPTRSV_ERROR_NOT_SUPPORTED = 5,  /* nnz >= 2^31, device is not sm_100, host_only plan solved, ... */
  SPTRSV_ERROR_ALLOC = 6,          /* device allocation failed */
  SPTRSV_ERROR_CUDA = 7,           /* CUDA runtime error (text in sptrsv_last_error) */
  SPTRSV_ERROR_DEADLOCK = 8        /* spin-wait watchdog tripped (reported by the next call on the plan) */
} sptrsv_status_t;

typedef enum { SPTRSV_R64F = 0, SPTRSV_R32F = 1 } sptrsv_dtype_t;
typedef enum { SPTRSV_LOWER = 0, SPTRSV_UPPER = 1 } sptrsv_fill_t;
typedef enum { SPTRSV_COL_MAJOR = 0, SPTRSV_ROW_MAJOR = 1 } sptrsv_layout_t;

/* Block variants of Sec 3.1: recursive (Alg 6, default), column (Alg 4), row (Alg 5). */
typedef enum { SPTRSV_VARIANT_REC = 0, SPTRSV_VARIANT_COL = 1, SPTRSV_VARIANT_ROW = 2 } sptrsv_variant_t;

/* Kernel labels of Alg 7 (names restored from L256/L258). */
typedef enum {
  SPTRSV_K_COMPLETELY_PARALLEL = 0, /* triangle with nlevels == 1 (L247 structure 1)  */
  SPTRSV_K_LEVEL_SET = 1,           /* (nnz/row==1 && nlevels<=100) || (nnz/row<=15 && nlevels<=20) */
  SPTRSV_K_SYNC_FREE = 2,           /* every other triangle (L256)                      */
  SPTRSV_K_NEAR_SERIAL = 3,         /* nlevels > 20000: the paper's cuSPARSE role (L256) */
  SPTRSV_K_SCALAR_CSR = 4,          /* square, nnz/row <= 12, emptyratio <= 50%         */
  SPTRSV_K_SCALAR_DCSR = 5,         /* square, nnz/row <= 12, emptyratio >  50%         */
  SPTRSV_K_VECTOR_CSR = 6,          /* square, nnz/row >  12, emptyratio <= 15%         */
  SPTRSV_K_VECTOR_DCSR = 7          /* square, nnz/row >  12, emptyratio >  15%         */
} sptrsv_kernel_t;

/* Storage format of a segment (L235-L241). */
typedef enum { SPTRSV_FMT_DIAG = 0, SPTRSV_FMT_CSR = 1, SPTRSV_FMT_DCSR = 2 } sptrsv_format_t;

/* The sm_100a kernel that actually executes a segment. */
typedef enum {
  SPTRSV_IMPL_TRI_DIAG = 0,      /* K1: x_i = b_i / d_i, elementwise                              */
  SPTRSV_IMPL_TRI_LEVELSET = 1,  /* K2: one multi-CTA launch per level (rows of a level contiguous) */
  SPTRSV_IMPL_TRI_SYNCFREE = 2,  /* K3: persistent multi-CTA, ticketed rows, per-row ready flags    */
  SPTRSV_IMPL_TRI_CHAIN = 3,     /* K4: single CTA, level loop with bar.sync, x window in smem      */
  SPTRSV_IMPL_SQ_SCALAR = 4,     /* K5/K7: thread (or RHS-group) per row, CSR or DCSR               */
  SPTRSV_IMPL_SQ_VECTOR = 5,     /* K6/K8: warp per row, CSR or DCSR                                */
  SPTRSV_IMPL_TRI_SUPERNODE = 6, /* B200: warp per fundamental supernode (<= 32 rows): dense GEMV of its
                                    shared external columns + register-resident dense triangle     */
  SPTRSV_IMPL_TRI_PIPE = 7,      /* B200: strand wavefront -- narrow-level triangle split by original row
                                    index into C x W strands (one warp each, one thread-block cluster);
                                    no level barrier; cross-strand x pushed into the consumer's shared
                                    memory (DSMEM).  Replaced by TRI_CHAIN at upload when a row has > 8
                                    dependencies (or > 10% would be polled in global memory)          */
  SPTRSV_IMPL_SQ_ADAPT = 8       /* B200: nnz-balanced row blocks (<= 32 rows, <= 256 entries) per warp,
                                    products staged in shared memory, lane-per-row sums; long rows
                                    alone (split into 1024-entry chunks with atomic partial sums)   */
} sptrsv_impl_t;

/* Which kernel implements each Alg 7 label. PAPER maps labels 1:1 onto the
 * kernels of L247-L250; B200 keeps the labels (parity) but lets a measured
 * cost model pick the sm_100a kernel per segment. */
typedef enum { SPTRSV_SELECT_PAPER = 0, SPTRSV_SELECT_B200 = 1 } sptrsv_selector_t;

typedef struct {
  int32_t variant;          /* sptrsv_variant_t, default REC                                   */
  int32_t depth;            /* -1 = the paper's rule (L299) -- under selector B200 with
                               min_block_rows 0, a root whose levels are all <= 2048 rows with
                               1..8 dependencies per row stays one triangle (R30);
                               >= 0 forces a uniform depth                                     */
  int64_t min_block_rows;   /* depth-rule threshold; 0 = 20 * SMs * 128 (378,880 on 148 SMs),
                               and 4x that under selector B200 with depth = -1 (DESIGN R33)   */
  int32_t reorder;          /* 0 = level-set reordering of every triangle (L231), 1 = none,
                               2 = auto (default): none when the input is supernodal (mean width of
                               its fundamental supernodes >= 8, R29), else level        */
  int32_t selector;         /* sptrsv_selector_t, default SPTRSV_SELECT_B200                   */
  int32_t force_tri_impl;   /* -1 = auto; else an sptrsv_impl_t for every triangle (tests)     */
  int32_t force_sq_impl;    /* -1 = auto; else an sptrsv_impl_t for every square (tests)       */
  int32_t host_only;        /* 1 = run the analysis only; no device memory; solve refused      */
  int32_t sm_count;         /* 0 = query the device (148 assumed when host_only)               */
  int32_t threads;          /* host threads for the analysis; 0 = hardware concurrency         */
  int32_t device;           /* CUDA device ordinal the plan lives on; -1 = the current device  */
  int32_t transpose;        /* 0 = the plan solves A x = b (default); 1 = it solves A^T x = b
                               for the given A (the preconditioner's transposed sweep, L33/L35;
                               SURVEY 8(f) f-4).  The given fill is validated as usual; the
                               system solved has the other fill (sptrsv_plan_info reports it).
                               The transpose is built on the host during the analysis; the solve
                               path is the one of an analysed A^T (R31).             */
  int32_t max_nrhs;         /* solve workspace sized at analysis for this many right-hand sides
                               (0 = allocated at the first solve that needs it)                 */
  int32_t graphs;           /* 1 (default) = a device solve whose (b, x, ldb, ldx, nrhs, layout)
                               repeats the previous uncaptured one is captured into a CUDA graph;
                               later solves with a captured key replay it (one graph launch).
                               0 = always launch the kernels one by one                        */
  int32_t analysis;         /* where sptrsv_analyse runs: 0 = auto (default):
                               on the device when row_ptr, col_idx and val are all device
                               pointers, else on the host; 1 = host; 2 = device (a host CSR is
                               copied to the device first).  Both give the same plan, bit for
                               bit (sptrsv_plan_hash).  The device analysis finishes on the host
                               when a segment's kernel needs a host-built format (strand
                               wavefront, TMA/ELL chain, supernode packing); it does not support
                               transpose = 1 (then the host analysis runs).  A device-analysed
                               plan keeps no host copy of P L P^T: sptrsv_plan_matrix returns
                               NOT_SUPPORTED for it.                                            */
  int32_t reserved[4];
  /* Device-memory hooks (SURVEY 8(b) "PyTorch for device memory"): when
   * dev_alloc is set, EVERY device allocation of the plan (arena, solve
   * workspace, flags, staging) goes through dev_alloc(bytes, stream, ctx) and
   * is returned by dev_free(ptr, stream, ctx); the Python binding passes the
   * torch CUDA caching allocator.  NULL = cudaMalloc / cudaFree.  dev_alloc
   * returns NULL on failure (SPTRSV_ERROR_ALLOC).  Both are called from the
   * thread calling sptrsv_analyse / sptrsv_solve / sptrsv_free, never during
   * graph capture or from device code. */
  void* (*dev_alloc)(size_t bytes, void* stream, void* ctx);
  void (*dev_free)(void* ptr, void* stream, void* ctx);
  void* alloc_ctx;
} sptrsv_opts_t;

/* Fill *o with the defaults above. */
void sptrsv_opts_default(sptrsv_opts_t* o);

/*
 * Preprocess L (or U) into a plan.  Blocking: on return the plan is usable on
 * any stream.
 *   n, nnz           matrix order and number of stored entries (nnz == row_ptr[n]).
 *   row_ptr[n+1],
 *   col_idx[nnz],
 *   val[nnz]         CSR, 0-based, columns strictly increasing in every row, the
 *                    diagonal present and non-zero (LOWER: last in its row, Alg 1
 *                    L65/L68; UPPER: first).  Host or device pointers (detected);
 *                    deep-copied: the caller may free them when the call returns.
 *   dtype            value type of val, b and x (fp64 or fp32; accumulation in dtype).
 *   fill             LOWER or UPPER; UPPER is solved as J U J (index reversal i -> n-1-i)
 *                    folded into the plan's permutation.
 *   opts             NULL = defaults.
 *   stream           used for the upload; synchronised before return.
 *   plan_out         receives the plan; set to NULL on any error.
 * Errors: INVALID_VALUE, NOT_TRIANGULAR, UNSORTED, ZERO_PIVOT (detail names the
 * row), NOT_SUPPORTED, ALLOC, CUDA.
 */
sptrsv_status_t sptrsv_analyse(int32_t n, int64_t nnz, const int32_t* row_ptr, const int32_t* col_idx,
                               const void* val, sptrsv_dtype_t dtype, sptrsv_fill_t fill,
                               const sptrsv_opts_t* opts, void* stream, sptrsv_plan_t* plan_out);

/*
 * Solve op(A) X = B for nrhs right-hand sides with a plan.
 *   b, ldb           B, nrhs columns of length n; COL_MAJOR: b[i + c*ldb] (ldb >= n),
 *                    ROW_MAJOR: b[i*ldb + c] (ldb >= nrhs).
 *   x, ldx           X, same conventions.  b == x (in place) is allowed.
 *   Device pointers: stream-ordered and asynchronous (no host synchronisation).
 *   Host pointers (both b and x in host memory): B is copied to the device,
 *   solved and X copied back inside this call, which then synchronises the
 *   stream (this is the end-to-end path bench.py times).
 *   Mixed host/device b and x is INVALID_VALUE.
 * One solve may be in flight per plan (the plan owns the solve workspace and
 * the per-row ready flags); concurrent use from two streams is undefined.
 * The first call for a given nrhs may allocate workspace (none when
 * opts.max_nrhs covers it).  With opts.graphs, the second consecutive device
 * solve with the same (b, x, ldb, ldx, nrhs, layout) captures the solve into
 * a CUDA graph and every later solve with that key is one graph launch
 * (at most 8 graphs are cached per plan, least recently used evicted).  If
 * the caller's stream is itself being captured, the kernels are enqueued
 * into the caller's capture instead.
 * b and x must live on the plan's device (INVALID_VALUE otherwise) and hold
 * the plan's dtype (not checkable here: the Python binding checks it).
 * Errors: INVALID_VALUE, NOT_SUPPORTED (host_only plan, non-sm_100 device),
 * ALLOC, CUDA, DEADLOCK (a watchdog of an EARLIER solve tripped).
 */
sptrsv_status_t sptrsv_solve(sptrsv_plan_t plan, const void* b, int64_t ldb, void* x, int64_t ldx,
                             int32_t nrhs, sptrsv_layout_t layout, void* stream);

/*
 * Solve A^T x = b with the plan of A (the preconditioner's
 * transposed sweep, PAPER.md:L33/L35 -- IC(0) applies L^{-T} L^{-1}), from
 * the SAME plan: no second analysis, no transposed copy of the matrix.
 * The plan stores L1 = D^-1 P A P^T (unit lower, R27), so
 * A^T x = b  <=>  L1^T z = P b, x = P^T D^-1 z.  L1^T is solved over the
 * plan's segments in reverse order with the push form of the sync-free solve
 * (Alg 3: in-degree counters decremented with atomics, left_sum
 * updated with atomicAdd; R32), squares as b_C -= S^T z_R with
 * atomics.  Summation order therefore varies run to run (reading R22).
 *   b, ldb, x, ldx, layout: as sptrsv_solve; nrhs must be 1 (NOT_SUPPORTED
 *   otherwise); b and x are DEVICE pointers on the plan's device
 *   (NOT_SUPPORTED for host pointers, INVALID_VALUE for another device).
 *   b == x is allowed.  Stream-ordered and asynchronous; never captured into
 *   a graph by the library.  The first call allocates 8n + 4*nseg bytes of
 *   counters (through dev_alloc when given) and builds them on the device.
 * A plan analysed with opts.transpose = 1 solves (A^T)^T = A here.
 * Errors: INVALID_VALUE, NOT_SUPPORTED, ALLOC, CUDA, DEADLOCK.
 */
sptrsv_status_t sptrsv_solve_transposed(sptrsv_plan_t plan, const void* b, int64_t ldb, void* x, int64_t ldx,
                                        int32_t nrhs, sptrsv_layout_t layout, void* stream);

/* Release the plan.  Waits for the plan's last solve (an event recorded on
 * that solve's stream) -- not for the whole device -- then returns every
 * device allocation (through dev_free when given).  NULL is a no-op. */
sptrsv_status_t sptrsv_free(sptrsv_plan_t plan);

/* ---------------------------------------------------------------- introspection
 * Used for the bit-exact structural parity against the oracle and for reporting. */
typedef struct {
  int32_t n, depth, nseg, variant, dtype, fill, reorder /* effective: 0 level, 1 none */, selector;
  int64_t nnz;
  int64_t min_block_rows;
  int32_t sm_count;
  int32_t launches_per_solve; /* kernel launches of one nrhs=1 solve (graph nodes)          */
  double analyse_ms;          /* host wall time of sptrsv_analyse, upload included          */
  int64_t device_bytes;       /* device memory owned by the plan (arena, excl. workspace)  */
  int32_t depth_rule;         /* 0 = the paper's rule (L299), 1 = B200 retune (a root with
                                 only narrow levels stays whole: DESIGN.md R30), 2 = caller's,
                                 3 = the B200 threshold (R33) gave a shallower tree          */
  int32_t analysis;           /* where the analysis ran: 0 host, 1 device (f-2), 2 device levels /
                                 reorder / P L P^T + host-built kernel formats                */
} sptrsv_plan_info_t;

typedef struct {
  int32_t kind; /* 0 = TRI, 1 = SQ */
  int32_t row0, row1, col0, col1; /* rows [row0,row1) x cols [col0,col1) of P L P^T     */
  int64_t nnz;                    /* TRI counts the diagonal                            */
  int32_t nlevels;                /* TRI: level sets of the triangle; SQ: 0             */
  int32_t nnz_per_row;            /* floor(nnz / rows)                                  */
  int32_t empty_rows;             /* SQ: rows without entries; TRI: 0                   */
  int32_t kernel;                 /* sptrsv_kernel_t (Alg 7 label)                      */
  int32_t format;                 /* sptrsv_format_t                                    */
  int32_t impl;                   /* sptrsv_impl_t actually launched                    */
  int32_t max_level_rows;         /* TRI: rows of the widest level                      */
} sptrsv_seg_info_t;

enum { SPTRSV_ARRAY_IN_DEGREE = 0, SPTRSV_ARRAY_LEVEL_PTR = 1, SPTRSV_ARRAY_DCSR_ROWS = 2 };

sptrsv_status_t sptrsv_plan_info(sptrsv_plan_t plan, sptrsv_plan_info_t* out);
/* Copy up to cap segment descriptors (execution order); *count = nseg. */
sptrsv_status_t sptrsv_plan_segments(sptrsv_plan_t plan, sptrsv_seg_info_t* out, int32_t cap,
                                     int32_t* count);
/* host_new_to_old[k] = original row of permuted row k (n entries). */
sptrsv_status_t sptrsv_plan_perm(sptrsv_plan_t plan, int32_t* host_new_to_old);
/* host_leaf_level[k] = level of permuted row k inside its leaf triangle (n entries). */
sptrsv_status_t sptrsv_plan_levels(sptrsv_plan_t plan, int32_t* host_leaf_level);
/* Per-segment integer arrays: IN_DEGREE (TRI, off-diagonal count per local row),
 * LEVEL_PTR (TRI, nlevels+1 local offsets), DCSR_ROWS (SQ, local nonempty rows).
 * Copies min(cap, size) entries; *count = size.  INVALID_VALUE if not defined. */
sptrsv_status_t sptrsv_plan_seg_array(sptrsv_plan_t plan, int32_t seg, int32_t which, int32_t* host_out,
                                      int64_t cap, int64_t* count);
/* The permuted matrix P L P^T (J U J P^T for UPPER) as CSR: row_ptr[n+1],
 * col_idx[nnz], val[nnz] (dtype of the plan).  Any pointer may be NULL. */
sptrsv_status_t sptrsv_plan_matrix(sptrsv_plan_t plan, int64_t* row_ptr, int32_t* col_idx, void* val);

/* 64-bit FNV-1a digest of everything a solve depends on: n, nnz, dtype,
 * fill, depth, the permutation, every segment descriptor and every stored
 * array (row pointers, columns, values, DCSR rows, level pointers) and the
 * scaled diagonal.  The analysis is bit-deterministic, so replicated plans
 * on different ranks must agree (all_reduce MIN == MAX).
 * Host-only computation; works for host_only plans. */
sptrsv_status_t sptrsv_plan_hash(sptrsv_plan_t plan, uint64_t* out);

/* Per-segment timing of later solves with CUDA events (diagnostics/bench).
 * When on, sptrsv_solve records an event around every segment on its stream;
 * sptrsv_seg_times synchronises and returns milliseconds of the LAST solve:
 * ms[0] = permute-in, ms[1 + s] = segment s, ms[1 + nseg] = permute-out. */
sptrsv_status_t sptrsv_set_profiling(sptrsv_plan_t plan, int32_t on);
sptrsv_status_t sptrsv_seg_times(sptrsv_plan_t plan, float* ms, int32_t cap, int32_t* count);

const char* sptrsv_status_string(sptrsv_status_t s);
const char* sptrsv_last_error(void);
/* Library version string (build id). */
const char* sptrsv_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SPTRSV_H_ */
