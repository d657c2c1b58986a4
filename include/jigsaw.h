/*
 * jigsaw.h -- C ABI of libjigsaw.so, the B200 (sm_100a) hot path of
 *   "Jigsaw: Accelerating SpMM with Vector Sparsity on Sparse Tensor Core"
 *   (Zhang, Liu et al., ICPP '24).
 *
 * Problem statement: C = A x B, where A (M x K) is a
 * vector-pruned sparse fp16 matrix (1-D column vectors of width v) and
 * B (K x N) is a dense fp16 matrix.  A is prepared once by the
 * multi-granularity sparsity reorder (Alg. 1) into the reorder-aware
 * storage format; the product then runs on the sm_100a sparse tensor
 * cores (tcgen05.mma.sp, 2:4).
 *
 * Conventions for every call:
 *   - Plain C99 types only.  Device pointers are CUDA device addresses on the
 *     CURRENT device; host pointers are ordinary (pageable or pinned) memory.
 *   - Matrices are row-major fp16 (IEEE binary16) with the leading dimension
 *     equal to the column count: A has ld = K, B has ld = N, C has ld = N.
 *   - Errors never abort: a call returns a status (or NULL) and records it in a
 *     thread-local slot readable with jigsaw_last_status() /
 *     jigsaw_last_error_string().
 *   - Zero test (DESIGN.md R-Q3): an fp16 entry is a nonzero iff
 *     (bits & 0x7FFF) != 0; -0 and +0 are zeros.  Non-finite values are carried
 *     but are outside the numerical tolerance contract.
 */
#ifndef JIGSAW_H_
#define JIGSAW_H_

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define JIGSAW_API __attribute__((visibility("default")))
#else
#define JIGSAW_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct jigsaw_handle_s* jigsaw_handle_t; /* opaque, immutable after creation */
typedef struct CUstream_st* jigsaw_stream_t;     /* a cudaStream_t; NULL = legacy default stream */

typedef enum {
  JIGSAW_SUCCESS = 0,
  JIGSAW_ERROR_INVALID_VALUE = 1, /* null pointer, bad size, misaligned buffer, bad option */
  JIGSAW_ERROR_UNSUPPORTED = 2,   /* no sm_100 device, or an option not built into this library */
  JIGSAW_ERROR_OUT_OF_MEMORY = 3, /* device allocation failed */
  JIGSAW_ERROR_CUDA = 4,          /* a CUDA runtime/driver call failed (message attached) */
  JIGSAW_ERROR_WRONG_DEVICE = 5,  /* current device differs from the handle's device */
  JIGSAW_ERROR_INTERNAL = 6       /* a builder invariant failed (bug) */
} jigsaw_status_t;

#define JIGSAW_PANEL_AUTOTUNE (-1)

/* Residual handling for columns evicted by the reorder retry. */
typedef enum {
  JIGSAW_RESIDUAL_SPTC = 0, /* paper: evicted columns re-queued into later 2:4 tiles (default) */
  JIGSAW_RESIDUAL_DENSE = 1 /* evicted columns form a dense tail run on dense tensor cores */
} jigsaw_residual_mode_t;

/* Element type of C (jigsaw_options_t.c_dtype; fp16 in, fp32
 * accumulate; C rounded to fp16 (RN, the paper's cublasHgemm output) or kept fp32). */
typedef enum {
  JIGSAW_C_F16 = 0, /* C is fp16 (IEEE binary16), round-to-nearest-even from the fp32 accumulator (default) */
  JIGSAW_C_F32 = 1  /* C is fp32: the fp32 accumulator as is */
} jigsaw_c_dtype_t;

/* Row order of the panels (jigsaw_options_t.row_order). */
typedef enum {
  JIGSAW_ROWS_GIVEN = 0,     /* panels are consecutive rows of A as given (the paper, default) */
  JIGSAW_ROWS_CLUSTERED = 1  /* row-clustered panels: rows sorted by their nonzero count (descending,
                                ties by row index) before the panels are formed, so rows of similar
                                density share a panel and sparse panels have fewer nonzero columns
                                (smaller K_p, fewer tiles); the SpMM scatters C rows back */
} jigsaw_row_order_t;

typedef struct {
  int panel_rows;    /* rows per panel (the BLOCK_TILE analogue, R-Q5/R-Q6): 128 (one CTA per
                        panel; the default when opt is NULL), 256 (a CTA pair per panel:
                        tcgen05 cta_group::2, M = 256, each dense B tile staged once per
                        pair), 0 = auto (256 when M >= 4096, else 128) or -1 = autotune
                        (JIGSAW_PANEL_AUTOTUNE: build both the 128- and the 256-row format,
                        time one jigsaw_spmm of each on the device with N = autotune_n
                        columns of B, keep the faster; the timing is part of the reorder's
                        preprocessing time).  16, 32 and 64
                        (the paper's BLOCK_TILE sizes) build the format for
                        export / statistics only: jigsaw_spmm on such a handle returns
                        JIGSAW_ERROR_UNSUPPORTED (no tcgen05 M below 128 is built) */
  int residual_mode; /* jigsaw_residual_mode_t */
  int c_dtype;       /* jigsaw_c_dtype_t: element type of C for every product with this handle */
  int row_order;     /* jigsaw_row_order_t */
  int autotune_n;    /* panel_rows = -1: columns of the probe product (0 = 256); else must be 0 */
  int cc_max_nnz;    /* CUDA-core tiles (§4.7: "for sparser data tile ...
                        accelerate the sparser data tiles using CUDA cores"; DESIGN.md R-Q28):
                        Z >= 0.  A 2:4 tile of the canonical reorder (main or overflow) whose
                        nonzero count -- the nonzeros of A in the panel's rows and the tile's
                        real columns -- is <= Z leaves the tile list (the other tiles keep their
                        order); the nonzeros of its columns become the panel's CUDA-core
                        entries (panel row, column, value), which the SpMM epilogue multiplies
                        on CUDA cores into the same fp32 accumulator row before C is written.
                        0 (default): no CUDA-core tiles.  DENSE residual tiles are not
                        affected.  Must be < 2^24. */
  int reserved[2];   /* must be zero */
} jigsaw_options_t;

/* Statistics of a prepared matrix (jigsaw_get_info). */
typedef struct {
  int64_t M, K;            /* shape of A */
  int32_t v;               /* vector width given at reorder (recorded, not used: R-Q22) */
  int32_t panel_rows;      /* P */
  int32_t residual_mode;   /* jigsaw_residual_mode_t */
  int32_t device;          /* CUDA ordinal the handle lives on */
  int32_t c_dtype;         /* jigsaw_c_dtype_t */
  int32_t row_order;       /* jigsaw_row_order_t */
  int64_t npanels;         /* ceil(M / P) */
  int64_t ntiles;          /* sum_p T_p: 2:4 tiles of 16 logical columns */
  int64_t ndtiles;         /* sum_p D_p: dense residual tiles (DENSE mode) */
  int64_t overflow_tiles;  /* tiles beyond ceil(K_p/16) per panel (SPTC mode) */
  int64_t evictions;       /* total columns moved by the reorder retry */
  int64_t nnz;             /* nonzero entries of A */
  int64_t kp_total;        /* sum_p K_p (non-zero columns per panel) */
  int64_t max_tiles;       /* max_p T_p */
  int64_t nksteps;         /* sum_p ceil(T_p/2): sparse MMA k-steps (32 logical columns) */
  int64_t format_bytes;    /* canonical format size: per tile 16P + 2P + 64 B (DESIGN.md R-Q19) */
  int64_t device_bytes;    /* device memory held by the handle */
  double reorder_ms;       /* device time of the reorder/format build */
  int32_t cc_max_nnz;      /* jigsaw_options_t.cc_max_nnz the handle was built with */
  int32_t reserved0;
  int64_t cc_tiles;        /* sum_p of the tiles moved to the CUDA cores (not in ntiles) */
  int64_t cc_entries;      /* CUDA-core entries (nonzeros of those tiles' columns) */
} jigsaw_info_t;

/* Caller-allocated host buffers for jigsaw_export_format; any member may be
 * NULL (skipped).  Sizes come from jigsaw_get_info (P = panel_rows). */
typedef struct {
  int64_t* T;        /* [npanels]          2:4 tiles per panel */
  int64_t* D;        /* [npanels]          dense residual tiles per panel */
  int32_t* col_idx;  /* [ntiles][16]       columns in pop order; -1 = PAD (col_idx_array) */
  uint8_t* perm;     /* [ntiles][16]       MMA_TILE column order (block_col_idx_array) */
  int32_t* gather;   /* [ntiles][16]       col_idx[perm[j]], read back from the device layout */
  uint16_t* vals;    /* [ntiles][P][8]     kept fp16 bits, decoded from the device layout */
  uint16_t* meta;    /* [ntiles][P]        2:4 metadata, nibble q = i0+4*i1 (sptc_col_idx_array) */
  uint8_t* kind;     /* [ntiles]           0 = main tile, 1 = overflow tile */
  uint8_t* nevict;   /* [ntiles]           evictions performed while building that tile */
  int32_t* rcol;     /* [ndtiles][16]      DENSE mode residual columns, -1 = PAD */
  uint16_t* dvals;   /* [ndtiles][P][16]   DENSE mode residual fp16 bits */
  int32_t* rowmap;   /* [M]                row r of the (row-clustered) panels is row rowmap[r] of A
                                           and of C; the identity for JIGSAW_ROWS_GIVEN.  The other
                                           arrays describe the matrix A[rowmap] */
  int64_t* cc_T;     /* [npanels]          tiles moved to the CUDA cores per panel (cc_max_nnz) */
  int64_t* cc_eoff;  /* [npanels + 1]      panel p owns CUDA-core entries cc_eoff[p] .. cc_eoff[p+1] */
  int32_t* cc_row;   /* [cc_entries]       row of the entry within its panel, entries ordered by */
  int32_t* cc_col;   /* [cc_entries]       (row, column): column of A */
  uint16_t* cc_val;  /* [cc_entries]       fp16 bits of A at (row, column), nonzero */
} jigsaw_format_host_t;

/* ---------------------------------------------------------------- north-star calls */

/* Multi-granularity sparsity reorder + reorder-aware format, with the
 * default options (P = 128, SPTC residual).
 *   A : device pointer, fp16 row-major M x K (ld = K), read-only, borrowed for the
 *       duration of the call (the handle keeps no reference to it).
 *   M, K > 0;  v in {1, 2, 4, 8} with M % v == 0 (v is validated and recorded).
 * Runs on the current device, synchronously (returns after the build finished).
 * Returns a new handle, or NULL on error (see jigsaw_last_status()). */
JIGSAW_API jigsaw_handle_t jigsaw_reorder(const void* A, int64_t M, int64_t K, int v);

/* C = A x B on sparse tensor cores, beta = 0: every element of C is written
 * (rows of an all-zero panel are written as zeros).
 *   B : device pointer, fp16 row-major K x N (ld = N), 16-byte aligned.
 *   C : device pointer, row-major M x N (ld = N), 16-byte aligned; overwritten.
 *       fp16, or fp32 if the handle was built with c_dtype = JIGSAW_C_F32.
 *   N > 0, N % 8 == 0 (TMA needs 16-byte rows).
 * Asynchronous on `stream`, never synchronises the host or the device.
 * Launches that use the dynamic tile scheduler or split long units into k-range
 * pieces need a small device workspace (scheduler ticket, piece counters, fp32
 * partial tiles): on an ordinary stream it is a region owned by that stream,
 * taken from the library's stream-ordered pool the first time the stream needs
 * it (or needs more) and then reused; under stream capture it is a graph-owned
 * allocation node plus a memset node zeroing its counters, freed right after
 * the kernel node.  So the
 * handle stays immutable and calls may run concurrently on any number of
 * streams, and captured graphs may be replayed concurrently with each other and
 * with eager calls.  C must not alias B.  The kernel is launched with
 * programmatic stream serialization: it may start while the previous kernel of
 * `stream` drains, but reads B, writes C and touches its workspace only after
 * that kernel has completed (stream order is preserved); it lets the next
 * programmatic launch on `stream` start once its own last work unit is
 * scheduled.  JIGSAW_PDL=0 in the environment (read once at load) disables
 * this. */
JIGSAW_API jigsaw_status_t jigsaw_spmm(jigsaw_handle_t h, const void* B, int64_t N, void* C,
                            jigsaw_stream_t stream);

/* Releases the handle's device memory (synchronises the handle's device first).
 * NULL is a no-op. */
JIGSAW_API void jigsaw_free(jigsaw_handle_t h);

/* ---------------------------------------------------------------- support calls */

JIGSAW_API jigsaw_status_t jigsaw_last_status(void);       /* thread-local, last call's status */
JIGSAW_API const char* jigsaw_last_error_string(void);     /* thread-local, valid until the next call */
JIGSAW_API const char* jigsaw_version(void);               /* static string */

/* jigsaw_reorder with explicit options and stream (opt == NULL: defaults).
 * Synchronous like jigsaw_reorder; *out receives the handle (NULL on error). */
JIGSAW_API jigsaw_status_t jigsaw_reorder_ex(const void* A, int64_t M, int64_t K, int v,
                                  const jigsaw_options_t* opt, jigsaw_stream_t stream,
                                  jigsaw_handle_t* out);

/* jigsaw_reorder_ex for `count` matrices at once (a batch of independent
 * matrices, e.g. every layer of a model): As[i] device fp16 Ms[i] x Ks[i]
 * (ld = Ks[i]), vs[i], the same options for all.  The builds run concurrently
 * on internal streams of the current device (host worker threads, one build
 * each at a time), ordered after prior work on `stream`; synchronous.  On
 * success out[i] receives the handles; on error every handle built so far is
 * freed, out[] is all NULL and the first failure's status is returned. */
JIGSAW_API jigsaw_status_t jigsaw_reorder_batched(const void* const* As, const int64_t* Ms, const int64_t* Ks,
                                                  const int* vs, int count, const jigsaw_options_t* opt,
                                                  jigsaw_stream_t stream, jigsaw_handle_t* out);

/* Same as jigsaw_reorder_ex but A is a HOST pointer (copied to the device inside). */
JIGSAW_API jigsaw_status_t jigsaw_reorder_host(const void* A_host, int64_t M, int64_t K, int v,
                                    const jigsaw_options_t* opt, jigsaw_stream_t stream,
                                    jigsaw_handle_t* out);

JIGSAW_API jigsaw_status_t jigsaw_get_info(jigsaw_handle_t h, jigsaw_info_t* out);

/* Copies the canonical format to caller-allocated host buffers (synchronous).
 * gather/vals/meta are reconstructed from the DEVICE layout the kernel consumes,
 * so a layout bug shows up as a mismatch against the oracle. */
JIGSAW_API jigsaw_status_t jigsaw_export_format(jigsaw_handle_t h, jigsaw_format_host_t* out);

/* C = A x B with B and C in HOST memory (end-to-end path): copies B in, runs
 * jigsaw_spmm, copies C out, all on `stream`, then synchronises `stream`.
 * C_host holds M x N elements of the handle's c_dtype.  Device staging buffers
 * are taken from the library's stream-ordered pool, which afterwards keeps the
 * largest host-buffer call's staging + 256 MB reserved (at most 1/4 of the
 * device's memory) so repeated calls do not map memory again. */
JIGSAW_API jigsaw_status_t jigsaw_spmm_host(jigsaw_handle_t h, const void* B_host, int64_t N, void* C_host,
                                 jigsaw_stream_t stream);

/* `count` independent products Cs[i] = A_i x Bs[i] (handles on the same device),
 * as ONE grouped persistent k_spmm launch per 64 products of the same panel
 * height (the batch of independent matrices, C5a).  Buffers and semantics as
 * jigsaw_spmm, per product. */
JIGSAW_API jigsaw_status_t jigsaw_spmm_batched(const jigsaw_handle_t* hs, const void* const* Bs,
                                    const int64_t* Ns, void* const* Cs, int count,
                                    jigsaw_stream_t stream);

/* The batch of jigsaw_spmm_batched with every B and C in HOST memory (the
 * end-to-end path of a batch): Bs_host[i] is K_i x Ns[i] fp16 row-major,
 * Cs_host[i] M_i x Ns[i] fp16 row-major (overwritten).  The batch is cut into
 * chunks whose host->device copies, grouped SpMM launches and device->host
 * copies run on three streams of the handles' device, so the copy engines of
 * both directions and the SMs work at the same time; pinned host buffers are
 * needed for the copies to overlap (pageable memory is correct but serial).
 * Device staging comes from the stream-ordered pool (kept reserved as for
 * jigsaw_spmm_host) and is returned to it before the call returns; each call uses helper streams of its own (concurrent calls from
 * several host threads do not wait for each other).  Ordered after prior work
 * on `stream`; synchronous: returns after every C is in host memory.  Errors as jigsaw_spmm_batched; a failure
 * in a later chunk leaves earlier Cs written. */
JIGSAW_API jigsaw_status_t jigsaw_spmm_batched_host(const jigsaw_handle_t* hs, const void* const* Bs_host,
                                                    const int64_t* Ns, void* const* Cs_host, int count,
                                                    jigsaw_stream_t stream);

/* Number of kernels the last successful jigsaw_spmm issued per call (for launch
 * accounting in benchmarks); reorder kernels are not counted. */
JIGSAW_API int jigsaw_spmm_launches_per_call(jigsaw_handle_t h, int64_t N);

/* ---------------------------------------------------------------- diagnostics */

/* How the calling thread's most recent jigsaw_spmm / jigsaw_spmm_batched /
 * host-buffer call was launched (for tests and benchmarks). */
typedef struct {
  int32_t launches;              /* k_spmm launches of that call */
  int32_t tile_n;                /* N columns per work unit (MMA N) of the last launch */
  int32_t split_k;               /* CTAs of a split-K cluster (1 = none) */
  int32_t grid;                  /* CTAs launched */
  int32_t cta_pair;              /* 1: 256-row panels on CTA pairs (cta_group::2) */
  int32_t problems;              /* products in the last launch */
  int32_t work_items;            /* scheduled work items (units, k-range pieces, padding) */
  int32_t split_slots;           /* k-range pieces reduced through the workspace (0 = none) */
  int32_t dynamic_schedule;      /* 1: dynamic tile scheduler */
  int32_t graph_owned_workspace; /* 1: workspace was a graph allocation node (stream capture) */
  int32_t nsplit_items;          /* column slices of long units (N-split, no workspace) */
  int32_t reserved[5];
} jigsaw_launch_desc_t;
JIGSAW_API jigsaw_status_t jigsaw_last_launch(jigsaw_launch_desc_t* out);

/* Diagnostic override of the launch configuration for the CALLING thread's later
 * calls (tests reach every kernel variant with it); NULL or all-zero restores
 * the library's choice.  Fields: tile_n (0 or 32/64/128/256 columns per unit),
 * split_k (0 or 1/2/4/8: single products of 128-row panels on split-K clusters
 * of that size, tile 64 or 32), no_pieces (1: no k-range pieces in grouped
 * launches), host_chunks (0 = library choice: ~6 MB chunks, 2..16; else the chunk count of
 * jigsaw_spmm_batched_host), k_pieces (1: split long units of grouped launches
 * into k-range pieces reduced through the workspace, instead of the default
 * column slices).  Results are identical up to fp32 summation order. */
typedef struct {
  int32_t tile_n, split_k, no_pieces, host_chunks, k_pieces;
  int32_t reserved[3]; /* must be zero */
} jigsaw_launch_override_t;
JIGSAW_API jigsaw_status_t jigsaw_set_launch_override(const jigsaw_launch_override_t* o);

/* Per-CTA timeline of the most recent k_spmm launch, recorded only when the
 * environment variable JIGSAW_TRACE=1 was set when the library was loaded (read
 * once; otherwise nothing is recorded).  Copies up to
 * max_ctas records of 24 int64 each into `out` (host): slots 0-11 are SM clock
 * (clock64) stamps at fixed points of the kernel (entry, setup done, first A/E
 * copy, first B copies, first full stage, last MMA commit, accumulator ready,
 * sends done, reduction data ready, stores done, exit), 13 / 15 are
 * %globaltimer (ns) at exit / entry, 14 is the SM id; 16-23 are prologue /
 * teardown stamps (A/E producer: first unit fetched, decoded, gather list
 * issued; B producer: unit decoded, gather list landed; MMA warp: unit decoded;
 * 23: exit barrier passed).  max_ctas < 0 instead
 * copies the per-k-block timeline of CTAs 0..7 (8 x 6 x 32 int64: A/E copy
 * issued, B copies issued, stage full seen by the MMA thread, commit issued,
 * metadata copy issued, MMAs issued).
 * Synchronous.  Returns the number of records copied (0 if none, -1 on a CUDA
 * error). */
JIGSAW_API int jigsaw_debug_trace(int64_t* out, int max_ctas);

#ifdef __cplusplus
}
#endif
#endif /* JIGSAW_H_ */
