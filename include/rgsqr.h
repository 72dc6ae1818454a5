/*
 * rgsqr.h -- C ABI of the B200-native out-of-core recursive classical Gram-Schmidt QR.
 *
 * The operation (Zhang & Wu, ICPP'21, /root/reference/PAPER.md):
 *   factor a tall matrix A (m x n, m >= n, "m is the number of rows and n is the
 *   number of columns") into Q (orthonormal columns) and R (upper
 *   triangular) with A = Q R, by classical Gram-Schmidt
 *   (Eq. 1; CGS evaluation order PAPER.md:109) organised as the
 *   column-halving recursion of Eq. 2:
 *       [A1|A2] = [Q1|Q2] [[R11, R12], [0, R22]]
 *       A1 = Q1 R11;  R12 = Q1^T A2;  A2 <- A2 - Q1 R12;  A2 = Q2 R22.
 *   When A does not fit the device-memory budget the two products stream row
 *   tiles host<->device with the copies overlapped by the math.
 *
 * Conventions (all functions):
 *   - Return an int status: 0 = OK, > 0 = warning (outputs valid), < 0 = error
 *     (outputs unspecified; message via rgsqr_last_error).
 *   - Matrices are COLUMN-MAJOR. A, Q: element (i,j) at base[i + j*lda].
 *     R: n x n, element (i,j) at R[i + j*n] (ldr = n), binary32, strict lower
 *     triangle written as 0.
 *   - Element type of A and Q is set by `precision`:
 *       RGSQR_FP16   -> IEEE binary16 storage, fp16 tensor-core operands, fp32 accumulate
 *       RGSQR_BF16   -> bfloat16 storage,       bf16 operands,               fp32 accumulate
 *       RGSQR_TF32   -> binary32 storage,       tf32 operands,               fp32 accumulate
 *       RGSQR_TF32X3 -> binary32 storage,       3-pass split tf32 (hi*hi + hi*lo + lo*hi)
 *   - Stored-value rounding (Q, updated A2', R12 used as an MMA operand) is
 *     round-to-nearest-even (reading R5).
 *   - Ownership: the caller owns every buffer it passes; the library never frees
 *     or reallocates them.  The library owns all device memory it allocates: a few
 *     context-lifetime buffers (stats.ctx_device_bytes, ~3 MB) plus a single arena of
 *     the rest of `device_mem_budget` (0 = all free memory minus a 512 MiB reserve),
 *     so the budget is enforced by construction (NCCL's own buffers excepted).
 *   - Blocking: rgsqr_factor* return after Q and R are complete (host-synchronous).
 *     A handle is not thread-safe; use one handle per thread / per GPU.
 *   - Preconditions: 1 <= n <= m, lda >= m, lda*sizeof(elem) % 16 == 0, pointers
 *     16-byte aligned.  Violations return RGSQR_ERR_INVALID_ARG.  rgsqr_factor with
 *     m*sizeof(elem) % 16 != 0 stages A / Q through zero-padded pinned copies ([A; 0] = [Q; 0] R).
 *   - Rank deficiency (the paper assumes linearly independent columns,
 *     PAPER.md:103): if some r_jj <= m * u_fp32 * ||a_j|| (or is not finite),
 *     q_j = 0 and r_jj = 0 are written, the first such j is reported in
 *     rgsqr_stats.first_breakdown_col, and RGSQR_WARN_RANK_DEFICIENT is returned.
 */
#ifndef RGSQR_H
#define RGSQR_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct rgsqr_ctx* rgsqr_handle;

enum rgsqr_precision { RGSQR_FP16 = 0, RGSQR_BF16 = 1, RGSQR_TF32 = 2, RGSQR_TF32X3 = 3 };

enum rgsqr_status {
  RGSQR_OK = 0,
  RGSQR_WARN_RANK_DEFICIENT = 1,
  RGSQR_ERR_INVALID_ARG = -1,
  RGSQR_ERR_BUDGET_TOO_SMALL = -2,
  RGSQR_ERR_CUDA = -3,
  RGSQR_ERR_NCCL = -4,
  RGSQR_ERR_UNSUPPORTED = -5,
  RGSQR_ERR_HOST_MEM = -6
};

/* Option keys for rgsqr_set_option / rgsqr_get_option. */
enum rgsqr_option {
  RGSQR_OPT_LEAF_WIDTH = 1,     /* columns factored by the in-kernel CGS leaf (8..64, default 64) */
  RGSQR_OPT_TILE_ROWS_MIN = 2,  /* OOC row-tile ramp start (paper: 2048; default 4096) */
  RGSQR_OPT_TILE_ROWS_MAX = 3,  /* OOC row-tile cap (paper: 8192/16384; default 16384) */
  RGSQR_OPT_RING_DEPTH = 4,     /* K device slots per OOC stream ring (>= 2, default 3) */
  RGSQR_OPT_ALGO = 5,           /* 0 = recursive (Eq. 2, default), 1 = blocked with the
                                   paper's OOC GEMM tilings, 2 = fused blocked: panel resident, trailing
                                   matrix streamed in column blocks read and written once per panel */
  RGSQR_OPT_BLOCK_COLS = 6,     /* panel width b of the blocked algorithm (default 8192) */
  RGSQR_OPT_SERIALIZE = 7,      /* 1 = one stream, no overlap (the paper's "Synchronous" rows) */
  RGSQR_OPT_REUSE = 8,          /* 1 = QR-level data reuse, default 1 */
  RGSQR_OPT_LEAF_CTAS = 9,      /* CTAs of the leaf kernel (0 = automatic) */
  RGSQR_OPT_SPLITK = 10,        /* force split-K factor of the TN product (0 = automatic) */
  RGSQR_OPT_PROFILE = 11,       /* 1 = time every kernel with CUDA events (rgsqr_stats.kern_*) */
  RGSQR_OPT_REORTH = 12,        /* 1 = CGS2: every projection R12 = Q1^T A2, A2 -= Q1 R12 and every leaf
                                   panel factorization applied twice ("twice is enough"
                                   reorthogonalization; CGS2 is named with CGS at PAPER.md:109 as the
                                   stable relative, reading R22).
                                   R12 = R12' + S, R_leaf = S R'.  Default 0 (the paper's CGS) */
  RGSQR_OPT_PREFETCH = 13       /* 1 = an OOC node uploads its first K ring tiles of A2 while its
                                   left child is being factored (cross-operation overlap,
                                   PAPER.md:231-233; tiles then start at full height instead of
                                   the ramp).  Default 1 */
  ,RGSQR_OPT_FUSE_SMALL = 14    /* 1 = nodes with w1, w2 <= 128 (fp16/bf16, one GPU) run R12 = Q1^T A2
                                   and A2 -= Q1 R12 (Eq. 2) as one kernel that
                                   reads Q1 and A2 once; 0 = the separate TN / NN products.
                                   Default 1 = nodes with w1, w2 <= 64; 2 = also up to 128 (A2 in
                                   two halves; measured slower at m = 65536, kept for study) */
  ,RGSQR_OPT_SPLIT_PCT = 15     /* width of an OUT-OF-CORE node's left child in percent of the node
                                   (rounded to 64).  50 = "divide evenly its columns into two halves"
                                   (PAPER.md:115), the default; other values are a scheduling ablation
                                   (same factorization in exact arithmetic).  In-core nodes always halve */
  ,RGSQR_OPT_X3_CHAIN = 16      /* TF32X3 products: at most this many k-blocks (32 rows / columns each,
                                   per operand segment) accumulate in one tensor-core fp32 chain in TMEM;
                                   the chains are summed with round-to-nearest fp32 adds (registers for
                                   the inner product, the shared-memory C tile for the outer product),
                                   because the tensor core's accumulation error grows with the chain
                                   length (R25).  Default 2 (inner product; the outer product uses
                                   twice this); 0 = unbounded chains */
  ,RGSQR_OPT_COLCHUNK = 17      /* 1 = column-chunked out-of-core node (DAG lookahead across the OOC
                                   boundary; R26): when the left child is
                                   in-core and resident, A2 is uploaded in the column order the right
                                   child consumes, R12 = Q1^T A2 and A2 -= Q1 R12 are applied per column
                                   chunk, and the right child starts while later columns are still in
                                   flight; the columns that do not fit beside Q1 are projected first
                                   from the host and re-uploaded once Q1's memory is free.  0 = the
                                   row-tile streamed node.  Default 1 */
  ,RGSQR_OPT_EAGER_PCT = 18     /* column-chunked node: complete the Q1 projection when the right child's
                                   leaves reach this percentage of its left half (default 50) */
  ,RGSQR_OPT_CHUNK_MIB = 19     /* host path: MiB per column-chunk upload of an in-core or column-chunked
                                   node (the granularity at which the recursion waits for its columns and
                                   applies deferred products; >= 256 columns per product piece).  Default 32 */
  ,RGSQR_OPT_VSHARDS = 20       /* p > 1: virtual row shards on ONE GPU (rgsqr_factor_device only; m must
                                   split into p equal 16-byte aligned row blocks): the arithmetic of a p-GPU
                                   row-sharded run -- every inner product as p local products (each with its
                                   own split-K) summed in shard order, every leaf's round-0 vector as p local
                                   vectors summed in shard order, no fused bottom node -- for testing the
                                   multi-GPU algebra without p GPUs.  Default 1 */
  ,RGSQR_OPT_DEFER_PIECES = 21  /* host path: a node whose columns are still uploading applies its deferred
                                   products (R23) in pieces of ~1/p of its A2 (p > 0) instead of
                                   one upload chunk (0, default): fewer, wider GEMMs vs an earlier start */
  ,RGSQR_OPT_PHASEA_PCT = 22    /* column-chunked node: percentage of the right child's first half whose Q1
                                   projection is applied before the right child starts (phase A, while the
                                   tail goes out; default 50) */
  ,RGSQR_OPT_GRAPH = 23         /* 1 (default): replay repeated rgsqr_factor / rgsqr_factor_device calls as one
                                   CUDA graph (captured on the first call with a given signature: buffers,
                                   shape, precision, budget, options, stream).  Host path: only when A, Q and
                                   R are already page-locked (rgsqr_host_alloc / cudaHostAlloc /
                                   cudaHostRegister) -- the captured copies address them directly.  Single-GPU
                                   contexts; off while RGSQR_OPT_PROFILE is set.  0: eager launches */
};

/* Counters of the last rgsqr_factor* call (bytes are host<->device link bytes). */
typedef struct rgsqr_stats {
  int64_t h2d_bytes;            /* all host->device bytes */
  int64_t d2h_bytes;            /* all device->host bytes */
  int64_t h2d_matrix_bytes;     /* A / A2' / Q words moved host->device */
  int64_t d2h_matrix_bytes;     /* Q / A2' words moved device->host */
  int64_t d2h_r_bytes;          /* R blocks moved device->host */
  int64_t d2d_bytes;            /* device-to-device staging copies */
  double  wall_ms;              /* host wall time of the factorization call */
  double  h2d_busy_ms;          /* sum of H2D copy durations (CUDA events) */
  double  d2h_busy_ms;          /* sum of D2H copy durations */
  double  compute_busy_ms;      /* sum of compute-stream segment durations */
  double  overlap_ratio;        /* (sum busy - wall) / (sum busy - max busy), R18 */
  double  pin_ms;               /* cudaHostRegister time (excluded from wall_ms) */
  int64_t arena_bytes;          /* size of the device arena */
  int64_t arena_high_water;     /* peak arena bytes in use */
  int64_t n_leaf_launches;
  int64_t n_tn_launches;
  int64_t n_nn_launches;
  int64_t n_other_launches;
  int64_t n_ooc_nodes;
  int64_t n_incore_nodes;
  int64_t first_breakdown_col;  /* -1 if none */
  int64_t flops;                /* 2 m n^2 (BASELINE.json metric convention) */
  /* Per-kernel-class accounting, filled only when RGSQR_OPT_PROFILE = 1 (CUDA events
   * around every launch).  Index: 0 leaf CGS, 1 inner product (TN + split-K reduce),
   * 2 outer product (NN), 3 other.  flops / bytes are ALGORITHMIC:
   *   leaf  (m x w):        2 m w^2 flop;          (2 m w) s + 4 w^2 bytes
   *   inner (w1, m, w2):    2 m w1 w2 flop;        m (w1 + w2) s + 4 w1 w2 bytes
   *   outer (m, w1, w2):    2 m w1 w2 flop;        m w1 s + w1 w2 s + 2 m w2 s bytes */
  double  kern_ms[4];
  int64_t kern_launches[4];
  double  kern_flops[4];
  double  kern_bytes[4];
  int64_t n_colchunk_nodes;     /* out-of-core nodes run column-chunked (RGSQR_OPT_COLCHUNK) */
  int64_t colchunk_tail_cols;   /* columns of those nodes projected from the host before the right
                                   child (they did not fit beside Q1) */
  int64_t ctx_device_bytes;     /* context-lifetime device buffers (leaf exchange words, partials, ...):
                                   counted against device_mem_budget, arena_bytes + this <= budget */
  int64_t graph_replay;         /* 1: this call ran as a CUDA graph (RGSQR_OPT_GRAPH); the per-stream busy
                                   times and overlap_ratio are then not measured (0) */
  int64_t graph_captures;       /* graphs captured by this handle so far */
} rgsqr_stats;

/* ---- lifetime -------------------------------------------------------------------- */
int rgsqr_create(rgsqr_handle* h, int device);
/* Multi-GPU (row-sharded, one process per GPU): rank 0 calls rgsqr_get_unique_id and
 * broadcasts the 128 bytes; every rank then calls rgsqr_create_dist collectively. */
int rgsqr_get_unique_id(unsigned char id[128]);
int rgsqr_create_dist(rgsqr_handle* h, int device, int rank, int nranks, const unsigned char id[128]);
int rgsqr_destroy(rgsqr_handle h);

/* ---- the factorization ------------------------------------------------------------- */
/* Host-resident out-of-core recursive CGS QR.  A_host: m x n (lda), host memory
 * (pinned or pageable; pageable buffers are page-locked for the call, cost in
 * stats.pin_ms).  Q_out: host, same element type and lda; may alias A_host (in
 * place).  R_out: host n x n binary32 (rank 0 only when nranks > 1; others may pass
 * NULL).  device_mem_budget: bytes of device memory the library may use (0 = all).
 * With nranks > 1, m is the number of LOCAL rows of this rank's contiguous row block. */
int rgsqr_factor(rgsqr_handle h, const void* A_host, int64_t lda, int64_t m, int64_t n,
                 void* Q_out, float* R_out, int precision, size_t device_mem_budget);

/* Same factorization with A, Q and R already resident in device memory (HBM).
 * A_dev / Q_dev: device pointers (Q_dev may alias A_dev), R_dev: device n x n
 * binary32.  device_mem_budget bounds the library's workspace only.  Runs on the
 * handle's stream (rgsqr_set_stream). */
int rgsqr_factor_device(rgsqr_handle h, const void* A_dev, int64_t lda, int64_t m, int64_t n,
                        void* Q_dev, float* R_dev, int precision, size_t device_mem_budget);

/* ---- the two out-of-core GEMMs as standalone operations (host memory in and out) ----------
 * The paper measures them separately (section 5.1, Tables 1/2) with both tiling
 * strategies of section 3.3:
 *   tiling 0 = recursive: inner product Fig. 3 (row tiles of Q1 and A2, each read once, R12
 *              accumulated in HBM and written once); outer product Fig. 5 (R12 resident, row tiles of
 *              Q1 and A2 in, A2' out).  `block` = rows per tile (0: 16384 inner, 8192 outer).
 *   tiling 1 = blocking:  inner product Fig. 4 (Q1 panel resident, A2 in column blocks, R12 blocks
 *              out); outer product Fig. 6 (Q1 and R12 resident, block x block tiles of A2 in and out).
 *              `block` = columns (inner) / tile edge (outer) (0: 16384).
 * Arrays are column-major host buffers (pageable ones are page-locked for the call): Q1 m x w1
 * (ldq), A2 m x w2 (lda) with the precision's storage type, R12 w1 x w2 binary32 (ldr >= w1).
 * Inner: R12 = Q1^T A2 (A2 read only).  Outer: A2 <- A2 - Q1 R12, R12 rounded RN to the operand
 * type on the device (R9), A2' rounded RN to storage.  device_mem_budget as for
 * rgsqr_factor.  FP16 / BF16 / TF32, single-GPU contexts; RGSQR_OPT_SERIALIZE gives the paper's "Synchronous" rows and
 * RGSQR_OPT_RING_DEPTH the number of tile slots.  Stats: bytes, busy times, overlap, wall_ms. */
int rgsqr_ooc_inner(rgsqr_handle h, const void* Q1_host, int64_t ldq, const void* A2_host, int64_t lda, int64_t m,
                    int64_t w1, int64_t w2, float* R12_host, int64_t ldr, int precision, int tiling, int64_t block,
                    size_t device_mem_budget);
int rgsqr_ooc_outer(rgsqr_handle h, const void* Q1_host, int64_t ldq, const float* R12_host, int64_t ldr,
                    void* A2_host, int64_t lda, int64_t m, int64_t w1, int64_t w2, int precision, int tiling,
                    int64_t block, size_t device_mem_budget);

/* ---- hot-path operations (device pointers; used by the kernel parity tests) ------------ */
/* Leaf CGS panel (Eq. 1) in place: P (m x w, ldp) -> Q; R11 (w x w,
 * device, ldr) receives r_ij, 1 <= w <= 64.  Returns the first breakdown column via
 * *breakdown (host int, -1 if none). */
int rgsqr_op_leaf(rgsqr_handle h, void* P, int64_t ldp, int64_t m, int64_t w,
                  float* R11, int64_t ldr, int precision, int* breakdown);
/* Inner product R12 (+)= Q1^T A2: Q1 m x w1 (ldq), A2 m x w2 (lda),
 * R12 binary32 w1 x w2 (ldr).  accumulate = 0: R12 = Q1^T A2; 1: R12 += Q1^T A2.
 * R12op (optional, may be NULL): R12 rounded to the operand type, ld = w1. */
int rgsqr_op_inner(rgsqr_handle h, const void* Q1, int64_t ldq, const void* A2, int64_t lda,
                   int64_t m, int64_t w1, int64_t w2, float* R12, int64_t ldr,
                   void* R12op, int accumulate, int precision);
/* Outer product A2 <- A2 - Q1 R12op: Q1 m x w1 (ldq), R12op
 * w1 x w2 operand-typed (ld = ldr), A2 m x w2 (lda) updated in place. */
int rgsqr_op_outer(rgsqr_handle h, const void* Q1, int64_t ldq, const void* R12op, int64_t ldr,
                   void* A2, int64_t lda, int64_t m, int64_t w1, int64_t w2, int precision);

/* ---- support ------------------------------------------------------------------------ */
int rgsqr_set_stream(rgsqr_handle h, void* cuda_stream);      /* NULL = library's own stream */
int rgsqr_get_stream(rgsqr_handle h, void** cuda_stream);
/* Pinned host memory on the GPU's NUMA node (sysfs numa_node of the GPU's PCI device): the pages
 * are first-touched by threads bound to that node's CPUs, then page-locked (cudaHostRegister).
 * Row shards of a multi-GPU run should live in their GPU's node.  Free with
 * rgsqr_host_free on the same handle (or rgsqr_destroy frees what is left). */
int rgsqr_host_alloc(rgsqr_handle h, size_t bytes, void** p);
int rgsqr_host_free(rgsqr_handle h, void* p);
int rgsqr_set_option(rgsqr_handle h, int key, int64_t value);
int rgsqr_get_option(rgsqr_handle h, int key, int64_t* value);
int rgsqr_get_stats(rgsqr_handle h, rgsqr_stats* out);
/* Host-link probe with the executor's own copy calls (cudaMemcpy2DAsync on the library's H2D and
 * D2H streams): `reps` copies of a rows x cols tile of elem_bytes-sized elements whose columns are
 * ld elements apart in the caller's pinned host buffer `host` (>= ld * cols elements), H2D alone,
 * D2H alone, then both directions concurrently.  gbps[0..2] = H2D, D2H and duplex-total GB/s
 * (10^9 B/s), CUDA-event timed.  The device tile is a temporary allocation outside any budget. */
int rgsqr_probe_link(rgsqr_handle h, void* host, int64_t ld, int64_t rows, int64_t cols, int elem_bytes,
                     int reps, double* gbps);
int rgsqr_version(void);                                        /* 100 * major + minor */
const char* rgsqr_status_string(int status);
const char* rgsqr_last_error(rgsqr_handle h);

#ifdef __cplusplus
}
#endif
#endif /* RGSQR_H */
