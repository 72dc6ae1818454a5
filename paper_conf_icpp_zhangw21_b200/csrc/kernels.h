// kernels.h -- internal launch interface of the device kernels (not part of the C ABI).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>

namespace rgsqr {

constexpr int LEAF_MAX_W = 64;
constexpr int LEAF_MAX_G = 160;       // leaf grid size cap (>= SM count)
// arrivals one exchange word can count (11-bit field, leaf.cu FX_CNT_SHIFT = 53): the leaf grid
// of a row-sharded run is capped at LEAF_MAX_ARRIVALS / nranks CTAs per GPU
constexpr int LEAF_MAX_ARRIVALS = 2047;
constexpr int LEAF_PARTS = 4;         // row quarters of the per-CTA partial sums
// leaf exchange words: [LEAF_XW_SETS round sets][LEAF_MAX_W+2 values], word i at
// xw[i * LEAF_XW_STRIDE] (one 256-byte line each: concurrent atomics and polls of different
// values land in different L2 slices)
constexpr int LEAF_XW_SETS = 8;
constexpr int LEAF_XW_STRIDE = 32;
constexpr int LEAF_XW_WORDS = LEAF_XW_SETS * (LEAF_MAX_W + 2);
constexpr size_t LEAF_SMEM_BUDGET = 200 * 1024;
// the leaf keeps its projected columns w_j in a ring of LEAF_WRING extra smem columns (the
// original a_j stay intact until u_j replaces them, see leaf.cu)
constexpr int LEAF_WRING = 3;
// rows per CTA the leaf's critical group holds in registers (8 rows x 256 threads)
constexpr int LEAF_MAX_RP = 2048;
// rows per CTA of a "tall" leaf panel (row state in shared memory, leaf.cu NR == 0): 8192 x 148 SMs
// = 1.2M rows on one GPU (configs[3] at p = 1); the panel width then shrinks to what fits on chip
constexpr int LEAF_MAX_RP_TALL = 8192;
// smem column stride of the leaf panel slice: >= rows and == 4 (mod 32), so that the
// float4 reads of 8 threads at the same row in 8 different columns hit 32 distinct banks
__host__ __device__ inline int leaf_ld(int rows) { return ((rows + 31) / 32) * 32 + 4; }

struct GemmParams {
  int64_t M, N, K;          // D[M x N] = sum_k A[M x K] B[N x K]^T (see gemm.cu)
  int64_t kb_total;         // K blocks of gemm_block_k() elements
  int64_t kb_per_split;     // K blocks per grid.z slice
  // inner product (TN) epilogue
  float* C;                 // fp32 output, ldc
  int64_t ldc;
  int accumulate;           // C += result
  void* Cop;                // optional operand-typed copy, ldop
  int64_t ldop;
  float* P;                 // split-K partials (non-null => write partials instead of C)
  int64_t ldp;
  int64_t split_stride;
  // outer product (NN) epilogue: A2 <- A2 - result
  void* A2;
  int64_t lda2;
  int64_t kb_seg;           // > 0: K blocks per operand segment (TF32X3: hi.lo, lo.hi, hi.hi)
};
// Launch-side extras of the TN/NN GEMM launches (kept out of GemmParams: its layout is the kernel's
// parameter block, and growing it measurably changed gemm_kernel's code generation)
struct GemmExtra {
  int group_m = 0;          // > 1: grouped tile rasterization, this many M-tiles per group (gemm.cu)
  int64_t kb_per_unit = 0;  // > 0 (fp32 TN only): k-blocks per tensor-core accumulation chain, the
                            // chains summed in fp64 registers (tn_promote_kernel, R25)
};

struct NNParams {
  int tiles_m, tiles_n;     // 128-row x BN-column output tiles
  int64_t kb_total;         // K blocks (K = w1; 3 x that for the TF32X3 segments)
  int64_t kb_seg;           // > 0: K blocks per operand segment (TF32X3: hi.lo, lo.hi, hi.hi)
  int64_t promote_kb;       // > 0: k-blocks per tensor-core accumulation chain, folded into the fp32
                            // C tile in between (fp32 storage only; R25)
};

// TF32X3: ma2 / mb2 are the lo operands of A / B; segments (A, B lo), (A lo, B), (A, B)
template <typename T>
cudaError_t launch_nn(int bn, const CUtensorMap& ma, const CUtensorMap& mb, const CUtensorMap& mc,
                      const NNParams& p, int grid, cudaStream_t st, const CUtensorMap* ma2 = nullptr,
                      const CUtensorMap* mb2 = nullptr);

struct LeafParams {
  void* P;                  // panel m x w (ldp), overwritten by Q
  int64_t ldp;
  int64_t m;
  int w;
  int rows_per_cta;
  float* R;                 // w x w block of R (ldr)
  int64_t ldr;
  float* partials;          // [2][LEAF_MAX_W+2][grid] per-CTA partial sums
  unsigned int* counter;    // grid barrier counter, never reset: round 0 waits for counter_target
  unsigned int counter_target;       // (set by the launcher from *counter_host)
  unsigned int* counter_host;        // host copy of the counter's value after all enqueued barriers
  long long* dbg;           // optional [w][8] clock64 stamps of CTA dbg_cta
  long long* dbg2;          // optional [grid][LEAF_MAX_W][2] globaltimer: critical publish, poll done
  int dbg_cta;
  int skip;                 // diagnostics only (RGSQR_LEAF_SKIP): 2 lookahead dots, 4 projection
  int poll_sleep_ns;        // backoff between exchange polls (RGSQR_LEAF_POLL_NS, default 0)
  int vec_ok;               // P and ldp*sizeof(elem) 16-byte aligned: vector panel loads
  unsigned int epoch;       // launch counter
  unsigned long long* xw;   // LEAF_XW_WORDS words (stride LEAF_XW_STRIDE), this GPU's, never reset
  unsigned long long* const* xw_peers;  // device array [nranks]: every GPU's xw (row-sharded run)
  unsigned long long* xprev_g;          // [LEAF_XW_WORDS] last-seen words, persistent
  int nranks;               // GPUs sharing the rows of the panel
  int sys;                  // distributed context: red.add into every rank's words, .sys scope
  int r0_mode;              // 0 round 0 in-kernel, 1 round-0-only (write r0buf), 2 round 0 given,
                            // 3 per-CTA round-0 partials already in `partials` (fused node)
  float* r0buf;             // [LEAF_MAX_W+2] round-0 vector (modes 1, 2)
  int64_t m_global;         // total rows (breakdown threshold)
  int* breakdown;           // device int, atomicMin of the first breakdown column
  int64_t col_offset;       // global index of the panel's first column
};

// fused bottom nodes (small.cu): R12 = Q1^T A2, A2 -= Q1 R12 for w1, w2 <= 128, fp16/bf16
struct SmallNodeParams {
  const void* Q1;
  int64_t ldq;
  void* A2;
  int64_t lda;
  int64_t m;
  int w1, w2;
  int rows_per_cta;         // multiple of 8
  int vec_ok;               // Q1/A2 16-byte aligned columns
  float* R12;               // fp32 out, ldr
  int64_t ldr;
  float* partials;          // [grid][W*W], W = 64 or 128
  void* r12op;              // [W][W] operand copy ([j][i])
  unsigned* counter;        // never reset: barrier k waits for counter_base + k G
  unsigned counter_base;    // (set by the launcher from *counter_host)
  unsigned* counter_host;   // host copy of the counter's value after all enqueued barriers
  float* r0_partials;       // non-null: also write the next leaf's round-0 partials of the new A2
                            // ([k][grid]: ||a_k||^2, k < w2, then a_0.a_1) -- leaf r0_mode 3
};
constexpr int SN_MAX_RP = 768;  // rows per CTA the fused bottom node holds in shared memory
size_t small_node_smem(int rp, int w);
template <typename T>
cudaError_t launch_small_node(const SmallNodeParams& p, int grid, cudaStream_t st);

int gemm_block_k(int elem_bytes);
int leaf_max_smem_rows(int w);

template <typename T>
cudaError_t launch_gemm(bool nn, int bn, const CUtensorMap& ma, const CUtensorMap& mb,
                        const GemmParams& p, int splits, cudaStream_t st, const CUtensorMap* ma2 = nullptr,
                        const CUtensorMap* mb2 = nullptr, GemmExtra x = GemmExtra{});
template <typename T>
cudaError_t launch_splitk_reduce(const float* P, int64_t split_stride, int64_t ldp, int splits,
                                 float* C, int64_t ldc, int accumulate, T* Cop, int64_t ldop,
                                 int64_t M, int64_t N, cudaStream_t st);
template <typename T>
cudaError_t launch_leaf(const LeafParams& p, int grid, cudaStream_t st);

// TF32X3 operand split: hi = RN_tf32(src), lo = RN_tf32(src - hi), M x N (R25)
cudaError_t launch_tf32_split(const float* src, int64_t lds, float* hi, int64_t ldh, float* lo, int64_t ldl,
                              int64_t M, int64_t N, int num_sms, cudaStream_t st);
// dst_f[i,j] = src[i,j] (optional) and dst_op[i,j] = RN(src[i,j]) (optional), M x N
template <typename T>
cudaError_t launch_copy_cast(const float* src, int64_t lds, float* dst_f, int64_t ldf, T* dst_op, int64_t ldo,
                             int64_t M, int64_t N, cudaStream_t st);

// R <- S R for upper-triangular w x w blocks (w <= LEAF_MAX_W), column-major, in place in R:
// the leaf's second CGS pass (CGS2) factors Q' = Q S, so A = Q' R' = Q (S R').
cudaError_t launch_trmm_upper(const float* S, int64_t lds, float* R, int64_t ldr, int w, cudaStream_t st);

}  // namespace rgsqr
