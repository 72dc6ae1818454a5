// ops.cu -- host launchers of the hot-path operations and the in-core recursion (Eq. 2).
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <climits>
#include <mutex>
#include <vector>

#include "engine.h"

namespace rgsqr {

int elem_bytes(int precision) { return (precision == RGSQR_FP16 || precision == RGSQR_BF16) ? 2 : 4; }

int fail(Ctx* c, int status, const std::string& msg) {
  if (c) c->last_error = msg;
  return status;
}

void Ctx::collect_kernel_stats() {
  for (auto& k : ksegs) {
    float ms = 0;
    cudaEventElapsedTime(&ms, k.a, k.b);
    stats.kern_ms[k.kind] += ms;
    stats.kern_launches[k.kind] += 1;
    stats.kern_flops[k.kind] += k.flops;
    stats.kern_bytes[k.kind] += k.bytes;
  }
  ksegs.clear();
}

cudaEvent_t Ctx::ev() {
  if (capturing) {
    // never-recorded events for a capture: a pooled event may still carry a record from an
    // earlier eager call, and waiting on it inside the capture would cross the capture boundary
    // (the executor waits on slot-free events before their first record: a no-op by design)
    cudaEvent_t e;
    cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
    capture_events.push_back(e);
    return e;
  }
  if (event_next == event_pool.size()) {
    cudaEvent_t e;
    cudaEventCreate(&e);
    event_pool.push_back(e);
  }
  return event_pool[event_next++];
}

// ---------------------------------------------------------------------------------
// TMA descriptors (driver entry point fetched through the runtime; no -lcuda)
// ---------------------------------------------------------------------------------
static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &p, 12000, cudaEnableDefault, &q) ==
            cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  });
  return fn;
}

bool encode_tmap_2d(CUtensorMap* map, int precision, const void* base, uint64_t inner, uint64_t outer,
                    uint64_t outer_stride_bytes, uint32_t box_inner, uint32_t box_outer, std::string* err,
                    int swz) {
  auto enc = get_encode();
  if (!enc) {
    *err = "cuTensorMapEncodeTiled unavailable";
    return false;
  }
  CUtensorMapDataType dt = precision == RGSQR_FP16   ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16
                           : precision == RGSQR_BF16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                                                     : CU_TENSOR_MAP_DATA_TYPE_FLOAT32;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {outer_stride_bytes};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(map, dt, 2, const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   swz == 1   ? CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B
                   : swz == 2 ? CU_TENSOR_MAP_SWIZZLE_NONE
                              : CU_TENSOR_MAP_SWIZZLE_128B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    *err = "cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ") dims=" + std::to_string(inner) + "x" +
           std::to_string(outer) + " stride=" + std::to_string(outer_stride_bytes);
    return false;
  }
  return true;
}

static int pick_bn(int64_t N) { return N >= 256 ? 256 : (N > 64 ? 128 : 64); }

template <typename T>
static int op_inner_local(Ctx* c, int prec, const void* Q1, int64_t ldq, const void* A2, int64_t lda, int64_t m,
                          int64_t w1, int64_t w2, float* R12, int64_t ldr, void* R12op, int64_t ldop,
                          int accumulate, cudaStream_t st);

// Row-sharded run: R12 = sum over ranks of the local Q1^T A2.  The local
// partial goes to a contiguous temporary, is summed with ncclAllReduce, and only then
// copied into R and rounded into the operand copy (the outer product and Q stay row-local).
template <typename T>
static int op_inner_t(Ctx* c, int prec, const void* Q1, int64_t ldq, const void* A2, int64_t lda, int64_t m,
                      int64_t w1, int64_t w2, float* R12, int64_t ldr, void* R12op, int64_t ldop, int accumulate,
                      cudaStream_t st, bool reduce_ranks) {
  if (!c->nccl_comm && c->opt.vshards > 1 && reduce_ranks) {
    // virtual row shards (RGSQR_OPT_VSHARDS): the multi-GPU arithmetic on one GPU --
    // every shard's local Q1_s^T A2_s (its own split-K), then the sum over shards in shard order
    const int64_t p = c->opt.vshards, ms = m / p;
    if (accumulate) return fail(c, RGSQR_ERR_UNSUPPORTED, "inner: accumulate with shard reduction");
    const size_t mark = c->arena.mark();
    float* tmp = static_cast<float*>(c->arena.alloc((size_t)p * w1 * w2 * sizeof(float)));
    if (!tmp) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "inner: no arena space for the shard partials");
    for (int64_t sh = 0; sh < p; ++sh) {
      const char* q = static_cast<const char*>(Q1) + sh * ms * (int64_t)sizeof(T);
      const char* a = static_cast<const char*>(A2) + sh * ms * (int64_t)sizeof(T);
      int rc = op_inner_local<T>(c, prec, q, ldq, a, lda, ms, w1, w2, tmp + sh * w1 * w2, w1, nullptr, 0, 0, st);
      if (rc < 0) return rc;
    }
    RGSQR_CUDA(c, launch_splitk_reduce<T>(tmp, w1 * w2, w1, (int)p, R12, ldr, 0, static_cast<T*>(R12op), ldop, w1,
                                          w2, st));
    c->stats.n_other_launches++;
    c->arena.release(mark);
    return RGSQR_OK;
  }
  if (!c->nccl_comm || !reduce_ranks)
    return op_inner_local<T>(c, prec, Q1, ldq, A2, lda, m, w1, w2, R12, ldr, R12op, ldop, accumulate, st);
  if (accumulate) return fail(c, RGSQR_ERR_UNSUPPORTED, "inner: accumulate with rank reduction");
  const size_t mark = c->arena.mark();
  float* tmp = static_cast<float*>(c->arena.alloc((size_t)w1 * w2 * sizeof(float)));
  if (!tmp) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "inner: no arena space for the R12 reduction");
  int rc = op_inner_local<T>(c, prec, Q1, ldq, A2, lda, m, w1, w2, tmp, w1, nullptr, 0, 0, st);
  if (rc < 0) return rc;
  rc = nccl_allreduce(c, tmp, (size_t)w1 * w2, NCCL_FLOAT32, st);
  if (rc < 0) return rc;
  RGSQR_CUDA(c, launch_copy_cast<T>(tmp, w1, R12, ldr, static_cast<T*>(R12op), ldop, w1, w2, st));
  c->stats.n_other_launches++;
  c->arena.release(mark);
  return RGSQR_OK;
}

template <typename T>
static int op_inner_once(Ctx* c, int prec, const void* Q1, int64_t ldq, const void* A2, int64_t lda, int64_t m,
                         int64_t w1, int64_t w2, float* R12, int64_t ldr, void* R12op, int64_t ldop,
                         int accumulate, cudaStream_t st, const void* Q1lo = nullptr, const void* A2lo = nullptr);

// TF32X3 (3-pass split tf32): Q1^T A2 ~= Q1h^T A2h + Q1h^T A2l + Q1l^T A2h with hi = RN_tf32(x),
// lo = RN_tf32(x - hi) (R25); the three products accumulate into R12 in one GEMM over
// three K segments, small terms first.  Error ~ |Q1l||A2l| <= 2^-22 relative per product.
template <typename T>
static int op_inner_local(Ctx* c, int prec, const void* Q1, int64_t ldq, const void* A2, int64_t lda, int64_t m,
                          int64_t w1, int64_t w2, float* R12, int64_t ldr, void* R12op, int64_t ldop,
                          int accumulate, cudaStream_t st) {
  if (prec != RGSQR_TF32X3)
    return op_inner_once<T>(c, prec, Q1, ldq, A2, lda, m, w1, w2, R12, ldr, R12op, ldop, accumulate, st);
  const size_t mark = c->arena.mark();
  const int64_t md = (m + 3) / 4 * 4;   // hi / lo leading dimension (16-byte TMA pitch)
  float* q_hi = static_cast<float*>(c->arena.alloc((size_t)md * w1 * 4));
  float* q_lo = static_cast<float*>(c->arena.alloc((size_t)md * w1 * 4));
  float* a_hi = static_cast<float*>(c->arena.alloc((size_t)md * w2 * 4));
  float* a_lo = static_cast<float*>(c->arena.alloc((size_t)md * w2 * 4));
  if (!q_hi || !q_lo || !a_hi || !a_lo)
    return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "inner (tf32x3): no space for the hi/lo operands");
  RGSQR_CUDA(c, launch_tf32_split(static_cast<const float*>(Q1), ldq, q_hi, md, q_lo, md, m, w1, c->num_sms, st));
  RGSQR_CUDA(c, launch_tf32_split(static_cast<const float*>(A2), lda, a_hi, md, a_lo, md, m, w2, c->num_sms, st));
  c->stats.n_other_launches += 2;
  // one GEMM over the three operand segments (K extended 3x): a single split-K reduction
  int rc = op_inner_once<T>(c, prec, q_hi, md, a_hi, md, m, w1, w2, R12, ldr, R12op, ldop, accumulate, st, q_lo, a_lo);
  c->arena.release(mark);
  return rc;
}

template <typename T>
static int op_inner_once(Ctx* c, int prec, const void* Q1, int64_t ldq, const void* A2, int64_t lda, int64_t m,
                         int64_t w1, int64_t w2, float* R12, int64_t ldr, void* R12op, int64_t ldop,
                         int accumulate, cudaStream_t st, const void* Q1lo, const void* A2lo) {
  const int s = (int)sizeof(T);
  const int BK = gemm_block_k(s);
  const bool promote = Q1lo != nullptr && A2lo != nullptr && c->opt.x3_chain > 0;
  const int bn = promote ? 128 : pick_bn(w2);   // (fp64 register accumulators: tn_promote_kernel)
  CUtensorMap ma, mb, ma2, mb2;
  std::string err;
  if (!encode_tmap_2d(&ma, prec, Q1, (uint64_t)m, (uint64_t)w1, (uint64_t)ldq * s, BK, 128, &err) ||
      !encode_tmap_2d(&mb, prec, A2, (uint64_t)m, (uint64_t)w2, (uint64_t)lda * s, BK, bn, &err))
    return fail(c, RGSQR_ERR_INVALID_ARG, "inner: " + err);
  const bool x3 = Q1lo != nullptr && A2lo != nullptr;
  if (x3 && (!encode_tmap_2d(&ma2, prec, Q1lo, (uint64_t)m, (uint64_t)w1, (uint64_t)ldq * s, BK, 128, &err) ||
             !encode_tmap_2d(&mb2, prec, A2lo, (uint64_t)m, (uint64_t)w2, (uint64_t)lda * s, BK, bn, &err)))
    return fail(c, RGSQR_ERR_INVALID_ARG, "inner (tf32x3): " + err);
  GemmParams p{};
  p.M = w1;
  p.N = w2;
  p.K = m;
  p.kb_total = (m + BK - 1) / BK;
  if (x3) {   // TF32X3: k-blocks of (Q1, A2 lo), (Q1 lo, A2), (Q1, A2): small terms first
    p.kb_seg = p.kb_total;
    p.kb_total *= 3;
  }
  const int64_t tiles = ((w1 + 127) / 128) * ((w2 + bn - 1) / bn);
  // grouped rasterization only pays on grids of many waves (e.g. the Table 1 shapes); on the
  // recursion's nodes (<= ~4 waves) the x-fastest order measured faster (RGSQR_GROUP_M overrides)
  static const int env_group = getenv("RGSQR_GROUP_M") ? atoi(getenv("RGSQR_GROUP_M")) : -1;
  GemmExtra gx;
  // (TF32X3's 128 x 128 fp32 tiles need ~128 B/clk/SM of operands: grouping 4 M-tiles keeps more of
  // them in L2 there, 108 -> 105 ms at configs[1]'s shape)
  // (16-bit, configs[1]'s top node: 16 M-tiles per group read 2.77x the algorithmic DRAM bytes vs 3.1x
  // x-fastest, at equal time -- profiles/r2_ncu_summary.md)
  gx.group_m = env_group >= 0 ? env_group
                              : (tiles > 2 * (int64_t)c->num_sms ? (x3 ? 4 : 16) : 0);
  // One wave: tiles x splits <= SMs (rounding up put 152 CTAs on 148 SMs at w1 = w2 = 512 and
  // doubled the kernel time: 57 vs 37 us, profiles/r1_splitk_scan.txt).
  int64_t splits = c->opt.splitk > 0 ? c->opt.splitk : (tiles >= c->num_sms ? 1 : c->num_sms / tiles);
  splits = std::max<int64_t>(1, std::min<int64_t>(splits, p.kb_total / 4));
  // TF32X3: the tensor-core accumulation chain is bounded in-kernel (RGSQR_OPT_X3_CHAIN k-blocks per
  // TMEM chain, the chains summed in fp32 registers: tn_promote_kernel, R25)
  if (x3) gx.kb_per_unit = c->opt.x3_chain;
  const size_t cap = std::min<size_t>((size_t)64 << 20, c->arena.free_bytes());
  while (splits > 1 && (size_t)splits * w1 * w2 * 4 + 256 > cap) --splits;
  p.kb_per_split = (p.kb_total + splits - 1) / splits;
  splits = (p.kb_total + p.kb_per_split - 1) / p.kb_per_split;
  if (p.kb_total == 0) {
    p.kb_per_split = 1;
    splits = 1;
  }
  size_t mark = c->arena.mark();
  cudaEvent_t kb = c->kbegin(st);
  if (splits > 1) {
    float* P = static_cast<float*>(c->arena.alloc((size_t)splits * w1 * w2 * sizeof(float)));
    if (!P) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "inner: no arena space for split-K partials");
    p.P = P;
    p.ldp = w1;
    p.split_stride = w1 * w2;
    RGSQR_CUDA(c, launch_gemm<T>(false, bn, ma, mb, p, (int)splits, st, x3 ? &ma2 : nullptr, x3 ? &mb2 : nullptr, gx));
    RGSQR_CUDA(c, launch_splitk_reduce<T>(P, w1 * w2, w1, (int)splits, R12, ldr, accumulate,
                                          static_cast<T*>(R12op), ldop, w1, w2, st));
    c->stats.n_other_launches++;
  } else {
    p.C = R12;
    p.ldc = ldr;
    p.accumulate = accumulate;
    p.Cop = R12op;
    p.ldop = ldop;
    RGSQR_CUDA(c, launch_gemm<T>(false, bn, ma, mb, p, 1, st, x3 ? &ma2 : nullptr, x3 ? &mb2 : nullptr, gx));
  }
  c->kend(1, st, kb, (x3 ? 6.0 : 2.0) * m * w1 * w2, (double)m * (w1 + w2) * s * (x3 ? 2 : 1) + 4.0 * w1 * w2);
  c->arena.release(mark);
  c->stats.n_tn_launches++;
  return RGSQR_OK;
}

template <typename T>
static int op_outer_t(Ctx* c, int prec, const void* Q1, int64_t ldq, const void* R12op, int64_t ldr, void* A2,
                      int64_t lda, int64_t m, int64_t w1, int64_t w2, cudaStream_t st, const void* Q1lo = nullptr,
                      const void* R12lo = nullptr) {
  const int s = (int)sizeof(T);
  const int BK = gemm_block_k(s);
  const int EPB = 128 / s;
  int bn = pick_bn(w2);
  if (s == 4) bn = std::min(bn, 128);  // fp32 C tile must leave room for the k-ring
  // short K (w1 <= 1024): the tile is bound by moving the old A2 tile in and A2' out; 128-wide
  // tiles leave room for two C buffers, so the next tile's load overlaps this tile's epilogue
  if (s == 2 && w1 <= 1024) bn = std::min(bn, 128);
  CUtensorMap ma, mb, mc;
  std::string err;
  // TMA needs 16-byte row pitches: a narrow node's R12 (w1 * s < 16 bytes, the 4-column leaves of tall
  // panels, R31) is copied to a padded scratch block first
  const size_t mark = c->arena.mark();
  if ((ldr * s) % 16 != 0) {
    const int64_t ldp = (w1 * s + 15) / 16 * 16 / s;
    void* pad = c->arena.alloc((size_t)ldp * w2 * s);
    if (!pad) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "outer: no space for the padded R12 operand");
    RGSQR_CUDA(c, cudaMemcpy2DAsync(pad, (size_t)ldp * s, R12op, (size_t)ldr * s, (size_t)w1 * s, (size_t)w2,
                                    cudaMemcpyDeviceToDevice, st));
    R12op = pad;
    ldr = ldp;
  }
  if (!encode_tmap_2d(&ma, prec, Q1, (uint64_t)m, (uint64_t)w1, (uint64_t)ldq * s, EPB, BK, &err, s == 4 ? 1 : 0) ||
      !encode_tmap_2d(&mb, prec, R12op, (uint64_t)w1, (uint64_t)w2, (uint64_t)ldr * s, BK, bn, &err) ||
      !encode_tmap_2d(&mc, prec, A2, (uint64_t)m, (uint64_t)w2, (uint64_t)lda * s, 128, 64, &err, 2)) {
    c->arena.release(mark);
    return fail(c, RGSQR_ERR_INVALID_ARG, "outer: " + err);
  }
  const bool x3 = Q1lo != nullptr && R12lo != nullptr;
  CUtensorMap ma2, mb2;
  if (x3 && (!encode_tmap_2d(&ma2, prec, Q1lo, (uint64_t)m, (uint64_t)w1, (uint64_t)ldq * s, EPB, BK, &err, s == 4 ? 1 : 0) ||
             !encode_tmap_2d(&mb2, prec, R12lo, (uint64_t)w1, (uint64_t)w2, (uint64_t)ldr * s, BK, bn, &err)))
  {
    c->arena.release(mark);
    return fail(c, RGSQR_ERR_INVALID_ARG, "outer (tf32x3): " + err);
  }
  NNParams p{};
  p.tiles_m = (int)((m + 127) / 128);
  p.tiles_n = (int)((w2 + bn - 1) / bn);
  p.kb_total = (w1 + BK - 1) / BK;
  if (x3) {   // TF32X3: k-blocks of (Q1, R12 lo), (Q1 lo, R12), (Q1, R12) into one accumulator
    p.kb_seg = p.kb_total;
    p.kb_total *= 3;
    // chains folded into the fp32 C tile (R25); twice the inner product's unit: K = w1 is
    // short, and a shorter unit would make the shared-memory C-tile updates the bound
    p.promote_kb = 2 * c->opt.x3_chain;
  }
  const int grid = (int)std::min<int64_t>((int64_t)p.tiles_m * p.tiles_n, c->num_sms);
  cudaEvent_t kb = c->kbegin(st);
  RGSQR_CUDA(c, launch_nn<T>(bn, ma, mb, mc, p, grid, st, x3 ? &ma2 : nullptr, x3 ? &mb2 : nullptr));
  c->kend(2, st, kb, (x3 ? 6.0 : 2.0) * m * w1 * w2,
          (double)m * w1 * s * (x3 ? 2 : 1) + (double)w1 * w2 * s * (x3 ? 2 : 1) + 2.0 * m * w2 * s);
  c->stats.n_nn_launches++;
  c->arena.release(mark);   // (stream-ordered reuse: later kernels on st run after this one)
  return RGSQR_OK;
}

int op_inner(Ctx* c, int prec, const void* Q1, int64_t ldq, const void* A2, int64_t lda, int64_t m, int64_t w1,
             int64_t w2, float* R12, int64_t ldr, void* R12op, int64_t ldop, int accumulate, cudaStream_t st,
             bool reduce_ranks) {
  switch (prec) {
    case RGSQR_FP16:
      return op_inner_t<__half>(c, prec, Q1, ldq, A2, lda, m, w1, w2, R12, ldr, R12op, ldop, accumulate, st,
                                reduce_ranks);
    case RGSQR_BF16:
      return op_inner_t<__nv_bfloat16>(c, prec, Q1, ldq, A2, lda, m, w1, w2, R12, ldr, R12op, ldop, accumulate, st,
                                       reduce_ranks);
    case RGSQR_TF32:
    case RGSQR_TF32X3:
      return op_inner_t<float>(c, prec, Q1, ldq, A2, lda, m, w1, w2, R12, ldr, R12op, ldop, accumulate, st,
                               reduce_ranks);
  }
  return fail(c, RGSQR_ERR_UNSUPPORTED, "inner: precision not supported");
}

int reduce_r12(Ctx* c, int prec, float* R12, int64_t ldr, void* R12op, int64_t ldop, int64_t w1, int64_t w2,
               cudaStream_t st) {
  if (ldr != w1) return fail(c, RGSQR_ERR_INVALID_ARG, "reduce_r12: R12 must be contiguous");
  if (c->nccl_comm) {
    int rc = nccl_allreduce(c, R12, (size_t)w1 * w2, NCCL_FLOAT32, st);
    if (rc < 0) return rc;
  }
  cudaError_t e;
  switch (prec) {
    case RGSQR_FP16:
      e = launch_copy_cast<__half>(R12, ldr, nullptr, 0, static_cast<__half*>(R12op), ldop, w1, w2, st);
      break;
    case RGSQR_BF16:
      e = launch_copy_cast<__nv_bfloat16>(R12, ldr, nullptr, 0, static_cast<__nv_bfloat16*>(R12op), ldop, w1,
                                          w2, st);
      break;
    default: e = launch_copy_cast<float>(R12, ldr, nullptr, 0, static_cast<float*>(R12op), ldop, w1, w2, st);
  }
  if (e != cudaSuccess) return fail(c, RGSQR_ERR_CUDA, std::string("reduce_r12: ") + cudaGetErrorString(e));
  c->stats.n_other_launches++;
  return RGSQR_OK;
}

int op_outer(Ctx* c, int prec, const void* Q1, int64_t ldq, const void* R12op, int64_t ldr, void* A2, int64_t lda,
             int64_t m, int64_t w1, int64_t w2, cudaStream_t st) {
  switch (prec) {
    case RGSQR_FP16: return op_outer_t<__half>(c, prec, Q1, ldq, R12op, ldr, A2, lda, m, w1, w2, st);
    case RGSQR_BF16: return op_outer_t<__nv_bfloat16>(c, prec, Q1, ldq, R12op, ldr, A2, lda, m, w1, w2, st);
    case RGSQR_TF32: return op_outer_t<float>(c, prec, Q1, ldq, R12op, ldr, A2, lda, m, w1, w2, st);
    case RGSQR_TF32X3: {
      // A2 <- A2 - (Q1h R12l + Q1l R12h + Q1h R12h): one NN pass over the three segments,
      // hi = RN_tf32(x), lo = RN_tf32(x - hi) (R25)
      const size_t mark = c->arena.mark();
      const int64_t md = (m + 3) / 4 * 4;    // 16-byte TMA pitch
      float* q_hi = static_cast<float*>(c->arena.alloc((size_t)md * w1 * 4));
      float* q_lo = static_cast<float*>(c->arena.alloc((size_t)md * w1 * 4));
      const int64_t lr = (w1 + 3) / 4 * 4;   // 16-byte TMA pitch
      float* r_hi = static_cast<float*>(c->arena.alloc((size_t)lr * w2 * 4));
      float* r_lo = static_cast<float*>(c->arena.alloc((size_t)lr * w2 * 4));
      if (!q_hi || !q_lo || !r_hi || !r_lo)
        return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "outer (tf32x3): no space for hi/lo operands");
      RGSQR_CUDA(c, launch_tf32_split(static_cast<const float*>(Q1), ldq, q_hi, md, q_lo, md, m, w1, c->num_sms, st));
      RGSQR_CUDA(c, launch_tf32_split(static_cast<const float*>(R12op), ldr, r_hi, lr, r_lo, lr, w1, w2, c->num_sms, st));
      c->stats.n_other_launches += 2;
      int rc = op_outer_t<float>(c, prec, q_hi, md, r_hi, lr, A2, lda, m, w1, w2, st, q_lo, r_lo);
      c->arena.release(mark);
      return rc;
    }
  }
  return fail(c, RGSQR_ERR_UNSUPPORTED, "outer: precision not supported");
}

// A TF32X3 recursion node, R12 = Q1^T A2 then A2 <- A2 - Q1 R12, with Q1 split into hi / lo ONCE for both
// products (op_inner + op_outer split it twice); same kernels and operands, so bitwise equal to the pair.
// Single-GPU contexts only (the row-sharded inner product reduces R12 across ranks first).
static int op_node_x3(Ctx* c, const void* Q1, int64_t ldq, void* A2, int64_t lda, int64_t m, int64_t w1, int64_t w2,
                      float* R12, int64_t ldr, void* R12op, cudaStream_t st) {
  const size_t mark = c->arena.mark();
  const int64_t md = (m + 3) / 4 * 4;   // hi / lo leading dimension (16-byte TMA pitch)
  float* q_hi = static_cast<float*>(c->arena.alloc((size_t)md * w1 * 4));
  float* q_lo = static_cast<float*>(c->arena.alloc((size_t)md * w1 * 4));
  const size_t mark_a = c->arena.mark();
  float* a_hi = static_cast<float*>(c->arena.alloc((size_t)md * w2 * 4));
  float* a_lo = static_cast<float*>(c->arena.alloc((size_t)md * w2 * 4));
  if (!q_hi || !q_lo || !a_hi || !a_lo) {
    c->arena.release(mark);
    return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "node (tf32x3): no space for the hi/lo operands");
  }
  RGSQR_CUDA(c, launch_tf32_split(static_cast<const float*>(Q1), ldq, q_hi, md, q_lo, md, m, w1, c->num_sms, st));
  RGSQR_CUDA(c, launch_tf32_split(static_cast<const float*>(A2), lda, a_hi, md, a_lo, md, m, w2, c->num_sms, st));
  c->stats.n_other_launches += 2;
  int rc = op_inner_once<float>(c, RGSQR_TF32X3, q_hi, md, a_hi, md, m, w1, w2, R12, ldr, R12op, w1, 0, st, q_lo, a_lo);
  if (rc < 0) {
    c->arena.release(mark);
    return rc;
  }
  c->arena.release(mark_a);   // (stream-ordered reuse: the outer product's buffers follow the inner product)
  const int64_t lr = (w1 + 3) / 4 * 4;
  float* r_hi = static_cast<float*>(c->arena.alloc((size_t)lr * w2 * 4));
  float* r_lo = static_cast<float*>(c->arena.alloc((size_t)lr * w2 * 4));
  if (!r_hi || !r_lo) {
    c->arena.release(mark);
    return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "node (tf32x3): no space for the R12 hi/lo operands");
  }
  RGSQR_CUDA(c, launch_tf32_split(static_cast<const float*>(R12op), w1, r_hi, lr, r_lo, lr, w1, w2, c->num_sms, st));
  c->stats.n_other_launches++;
  rc = op_outer_t<float>(c, RGSQR_TF32X3, q_hi, md, r_hi, lr, A2, lda, m, w1, w2, st, q_lo, r_lo);
  c->arena.release(mark);
  return rc;
}

static void leaf_geometry(Ctx* c, int64_t m, int* grid, int* rp) {
  int G = c->opt.leaf_ctas > 0 ? (int)c->opt.leaf_ctas : c->num_sms;
  G = (int)std::max<int64_t>(1, std::min<int64_t>({(int64_t)G, (int64_t)LEAF_MAX_G, (m + 31) / 32}));
  // the exchange word counts nranks x G arrivals in its top 11 bits (leaf.cu FX_CNT_SHIFT)
  G = std::max(1, std::min(G, LEAF_MAX_ARRIVALS / std::max(1, c->nranks)));
  int64_t r = (m + G - 1) / G;
  r = (r + 7) & ~int64_t(7);  // 16-byte aligned row slices for the vector loads
  *grid = G;
  *rp = (int)r;
}

int leaf_width_for(Ctx* c, int64_t m) {
  int G, rp;
  leaf_geometry(c, m, &G, &rp);
  if (rp > LEAF_MAX_RP_TALL) return 0;
  int64_t wmax = (int64_t)LEAF_SMEM_BUDGET / ((int64_t)leaf_ld(rp) * 4) - LEAF_WRING;
  int64_t w = std::min<int64_t>({c->opt.leaf_width, (int64_t)LEAF_MAX_W, wmax});
  if (w >= 8) w &= ~int64_t(7);
  return (int)w;
}

int op_leaf(Ctx* c, int prec, void* P, int64_t ldp, int64_t m, int64_t w, float* R11, int64_t ldr,
            int64_t col_offset, cudaStream_t st, bool r0_pre) {
  int G, rp;
  leaf_geometry(c, m, &G, &rp);
  if (rp > LEAF_MAX_RP_TALL)
    return fail(c, RGSQR_ERR_UNSUPPORTED, "leaf: " + std::to_string(m) + " rows exceed " +
                                              std::to_string(LEAF_MAX_RP_TALL) + " per CTA");
  if (w < 1 || w > LEAF_MAX_W || (size_t)(w + LEAF_WRING) * leaf_ld(rp) * 4 > LEAF_SMEM_BUDGET)
    return fail(c, RGSQR_ERR_UNSUPPORTED, "leaf: panel " + std::to_string(m) + "x" + std::to_string(w) +
                                              " does not fit on chip");
  LeafParams p{};
  p.P = P;
  p.ldp = ldp;
  p.m = m;
  p.w = (int)w;
  p.rows_per_cta = rp;
  p.R = R11;
  p.ldr = ldr;
  p.partials = c->d_partials;
  static const bool dbg = getenv("RGSQR_LEAF_DEBUG") != nullptr;
  static long long* dbg_buf = nullptr;
  p.counter = c->d_counter;
  p.counter_host = &c->counter_host[0];
  p.epoch = ++c->leaf_epoch;
  p.xw = c->d_xw;
  p.xw_peers = c->d_peers;
  p.xprev_g = c->d_xprev;
  p.nranks = c->nranks;
  p.sys = c->nccl_comm != nullptr;
  p.r0buf = c->d_r0buf;
  p.m_global = c->m_global > 0 ? c->m_global : m;
  p.vec_ok = ((ldp * elem_bytes(prec)) % 16 == 0) && (reinterpret_cast<uintptr_t>(P) % 16 == 0);
  if (dbg && !dbg_buf) cudaMalloc(&dbg_buf, sizeof(long long) * 16 * (LEAF_MAX_W + 1));
  p.dbg = dbg ? dbg_buf : nullptr;
  static const bool dbg2 = getenv("RGSQR_LEAF_DEBUG2") != nullptr;
  static long long* dbg2_buf = nullptr;
  if (dbg2 && !dbg2_buf) cudaMalloc(&dbg2_buf, sizeof(long long) * (2 * LEAF_MAX_W + 1) * LEAF_MAX_G);
  p.dbg2 = dbg2 ? dbg2_buf : nullptr;
  p.dbg_cta = dbg ? atoi(getenv("RGSQR_LEAF_DEBUG")) : 0;
  static const int skip = getenv("RGSQR_LEAF_SKIP") ? atoi(getenv("RGSQR_LEAF_SKIP")) : 0;
  p.skip = dbg ? skip : 0;
  static const int poll_ns = getenv("RGSQR_LEAF_POLL_NS") ? atoi(getenv("RGSQR_LEAF_POLL_NS")) : 0;
  p.poll_sleep_ns = poll_ns;
  p.breakdown = c->d_breakdown;
  p.col_offset = col_offset;
  auto launch = [&](const LeafParams& q) -> cudaError_t {
    switch (prec) {
      case RGSQR_FP16: return launch_leaf<__half>(q, G, st);
      case RGSQR_BF16: return launch_leaf<__nv_bfloat16>(q, G, st);
      case RGSQR_TF32:
      case RGSQR_TF32X3: return launch_leaf<float>(q, G, st);   // fp32 CUDA-core leaf either way
    }
    return cudaErrorInvalidValue;
  };
  if (prec < RGSQR_FP16 || prec > RGSQR_TF32X3)
    return fail(c, RGSQR_ERR_UNSUPPORTED, "leaf: precision not supported");
  cudaError_t e;
  cudaEvent_t kb = c->kbegin(st);
  if (!c->nccl_comm && c->opt.vshards > 1) {
    // virtual row shards: each shard's round-0 vector (column norms, a_0.a_1) from a round-0-only
    // launch over its rows, summed in shard order (the multi-GPU round-0 allreduce), then the main
    // launch over all rows with the given vector
    const int64_t ns = c->opt.vshards, ms = m / ns, L = LEAF_MAX_W + 2;
    const size_t mark = c->arena.mark();
    float* r0s = static_cast<float*>(c->arena.alloc((size_t)ns * L * sizeof(float)));
    if (!r0s) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "leaf: no arena space for the shard round-0 vectors");
    e = cudaSuccess;
    for (int64_t sh = 0; sh < ns && e == cudaSuccess; ++sh) {
      LeafParams p0 = p;
      int Gs, rps;
      leaf_geometry(c, ms, &Gs, &rps);
      p0.P = static_cast<char*>(P) + sh * ms * elem_bytes(prec);
      p0.m = ms;
      p0.rows_per_cta = rps;
      p0.r0_mode = 1;
      p0.r0buf = r0s + sh * L;
      e = [&]() -> cudaError_t {
        switch (prec) {
          case RGSQR_FP16: return launch_leaf<__half>(p0, Gs, st);
          case RGSQR_BF16: return launch_leaf<__nv_bfloat16>(p0, Gs, st);
          default: return launch_leaf<float>(p0, Gs, st);
        }
      }();
    }
    if (e == cudaSuccess)
      e = launch_splitk_reduce<float>(r0s, L, L, (int)ns, c->d_r0buf, L, 0, nullptr, 0, w + 1, 1, st);
    if (e == cudaSuccess) {
      p.r0_mode = 2;
      e = launch(p);
    }
    c->arena.release(mark);
  } else if (!c->nccl_comm) {
    p.r0_mode = r0_pre ? 3 : 0;
    e = launch(p);
  } else {
    // row-sharded: round 0 (column norms -> fixed-point scales) is summed over GPUs by NCCL
    // between a round-0-only launch and the main launch; later rounds reduce in-kernel
    LeafParams p0 = p;
    p0.r0_mode = 1;
    e = launch(p0);
    if (e == cudaSuccess) {
      int rc = nccl_allreduce(c, c->d_r0buf, (size_t)w + 1, NCCL_FLOAT32, st);
      if (rc < 0) return rc;
      p.r0_mode = 2;
      e = launch(p);
    }
  }
  if (e != cudaSuccess) return fail(c, RGSQR_ERR_CUDA, std::string("leaf launch: ") + cudaGetErrorString(e));
  const int s = elem_bytes(prec);
  c->kend(0, st, kb, 2.0 * m * w * w, 2.0 * m * w * s + 4.0 * w * w);
  if (p.dbg) {
    long long hb[16 * (LEAF_MAX_W + 1)];
    cudaMemcpyAsync(hb, p.dbg, sizeof(long long) * 16 * (LEAF_MAX_W + 1), cudaMemcpyDeviceToHost, st);
    cudaStreamSynchronize(st);
    // critical stamps of round t: 0 start, 1 exchanged, 2 scalars, 3 row pass + butterfly,
    // 4 group barrier, 7 published, 5 projection; bulk stamps: 13 before BAR_Q, 8 after,
    // 9 lookahead GEMV, 11 reduced, 12 end
    auto avg = [&](int a, int b, int t0, int t1) {
      double sacc = 0;
      int n = 0;
      for (int t = t0; t < t1; ++t, ++n) sacc += (double)(hb[t * 16 + b] - hb[t * 16 + a]);
      return n ? sacc / n : 0.0;
    };
    const int t0 = 2, t1 = (int)w - 5;
    double per = 0;
    for (int t = t0; t < t1; ++t) per += (double)(hb[(t + 1) * 16] - hb[t * 16]);
    per /= std::max(1, t1 - t0);
    fprintf(stderr,
            "[leaf m=%lld w=%lld G=%d RP=%d] cycles/round %.0f | critical: exchange %.0f scalars %.0f rowpass %.0f "
            "sync %.0f publish %.0f | bulk: wait %.0f gemv %.0f poll %.0f project %.0f busy %.0f\n",
            (long long)m, (long long)w, G, rp, per, avg(0, 1, t0, t1), avg(1, 2, t0, t1), avg(2, 3, t0, t1),
            avg(3, 4, t0, t1), avg(4, 7, t0, t1), avg(13, 8, t0, t1), avg(8, 9, t0, t1), avg(9, 10, t0, t1),
            avg(10, 11, t0, t1), avg(8, 12, t0, t1));
  }
  if (p.dbg) {
    long long pb[12];
    cudaMemcpyAsync(pb, p.dbg + 16 * LEAF_MAX_W, sizeof(long long) * 12, cudaMemcpyDeviceToHost, st);
    cudaStreamSynchronize(st);
    fprintf(stderr, "[leaf prologue/epilogue cycles] xprev+load %lld round0 %lld (dots %lld partials %lld barrier %lld "
            "gather %lld) tables %lld rounds %lld join %lld store %lld\n",
            pb[1] - pb[0], pb[2] - pb[1], pb[8] - pb[1], pb[9] - pb[8], pb[10] - pb[9], pb[2] - pb[10],
            pb[3] - pb[2], pb[4] - pb[3], pb[5] - pb[4], pb[6] - pb[5]);
  }
  if (p.dbg2) {
    std::vector<long long> hb((size_t)2 * LEAF_MAX_W * G);
    cudaMemcpyAsync(hb.data(), p.dbg2, sizeof(long long) * hb.size(), cudaMemcpyDeviceToHost, st);
    cudaStreamSynchronize(st);
    // exchange round r: published in iteration r-1 (slot 0), detected in iteration r (slot 1)
    double skew = 0, first = 0, last = 0, mean = 0, per = 0;
    int cnt = 0;
    for (int r = 2; r + 1 < w; ++r, ++cnt) {
      long long pmax = LLONG_MIN, pmin = LLONG_MAX, dmin = LLONG_MAX, dmax = LLONG_MIN;
      double dsum = 0;
      for (int g = 0; g < G; ++g) {
        const long long P = hb[((size_t)g * LEAF_MAX_W + r - 1) * 2], D = hb[((size_t)g * LEAF_MAX_W + r) * 2 + 1];
        pmax = std::max(pmax, P); pmin = std::min(pmin, P);
        dmax = std::max(dmax, D); dmin = std::min(dmin, D);
        dsum += (double)D;
      }
      skew += (double)(pmax - pmin);
      first += (double)(dmin - pmax);
      last += (double)(dmax - pmax);
      mean += dsum / G - (double)pmax;
      per += (double)(hb[((size_t)0 * LEAF_MAX_W + r) * 2] - hb[((size_t)0 * LEAF_MAX_W + r - 1) * 2]);
    }
    cnt = std::max(cnt, 1);
    {
      // which CTAs publish last / detect last, and each CTA's mean lateness behind the first publisher
      std::vector<int> lastp(G, 0), lastd(G, 0);
      std::vector<double> late(G, 0.0);
      for (int r = 2; r + 1 < w; ++r) {
        int gp = 0, gd = 0;
        long long pmin = LLONG_MAX;
        for (int q = 0; q < G; ++q) pmin = std::min(pmin, hb[((size_t)q * LEAF_MAX_W + r - 1) * 2]);
        for (int q = 0; q < G; ++q) {
          const long long P = hb[((size_t)q * LEAF_MAX_W + r - 1) * 2], D = hb[((size_t)q * LEAF_MAX_W + r) * 2 + 1];
          if (P > hb[((size_t)gp * LEAF_MAX_W + r - 1) * 2]) gp = q;
          if (D > hb[((size_t)gd * LEAF_MAX_W + r) * 2 + 1]) gd = q;
          late[q] += (double)(P - pmin);
        }
        lastp[gp]++;
        lastd[gd]++;
      }
      std::string sp = "", sd = "", sl = "";
      for (int q = 0; q < G; ++q) {
        if (lastp[q]) sp += " " + std::to_string(q) + ":" + std::to_string(lastp[q]);
        if (lastd[q]) sd += " " + std::to_string(q) + ":" + std::to_string(lastd[q]);
      }
      std::vector<int> ord(G);
      for (int q = 0; q < G; ++q) ord[q] = q;
      std::sort(ord.begin(), ord.end(), [&](int a2, int b2) { return late[a2] > late[b2]; });
      std::vector<long long> smid(G);
      cudaMemcpy(smid.data(), p.dbg2 + (size_t)2 * LEAF_MAX_W * LEAF_MAX_G, sizeof(long long) * G, cudaMemcpyDeviceToHost);
      for (int k = 0; k < G; ++k)
        sl += " " + std::to_string(ord[k]) + "/" + std::to_string(smid[ord[k]]) + ":" +
              std::to_string((int)(late[ord[k]] / std::max(1, cnt)));
      fprintf(stderr, "[leaf2] last publisher (cta:rounds)%s | last detector%s | mean publish lateness (cta/smid:ns, latest first)%s\n",
              sp.c_str(), sd.c_str(), sl.c_str());
      std::string late_sm = "";
      int nl = 0;
      for (int q = 0; q < G; ++q)
        if (late[q] / std::max(1, cnt) > 330.0) {
          ++nl;
          late_sm += " " + std::to_string(smid[q]);
        }
      fprintf(stderr, "[leaf2] late (> 330 ns) CTAs: %d, their SMs:%s\n", nl, late_sm.c_str());
    }
    fprintf(stderr, "[leaf2 m=%lld w=%lld G=%d] ns/round %.0f | publish skew %.0f | last publish -> detect: first %.0f mean %.0f last %.0f\n",
            (long long)m, (long long)w, G, per / cnt, skew / cnt, first / cnt, mean / cnt, last / cnt);
  }
  c->stats.n_leaf_launches++;
  return RGSQR_OK;
}

// fused bottom node (small.cu): returns 1 when done (2: and the right child leaf's round-0
// partials were written), 0 when the shape / precision / context is not covered (the caller
// then runs the separate products), < 0 on error
int op_small_node(Ctx* c, int prec, const void* Q1, int64_t ldq, void* A2, int64_t lda, int64_t m, int64_t w1,
                  int64_t w2, float* R12, int64_t ldr, cudaStream_t st, bool r0_for_leaf) {
  if (!c->opt.fuse_small || c->nccl_comm || c->opt.vshards > 1 || w1 > 128 || w2 > 128 || w1 < 1 || w2 < 1) return 0;
  if (prec != RGSQR_FP16 && prec != RGSQR_BF16) return 0;
  const int W = (w1 <= 64 && w2 <= 64) ? 64 : 128;
  if (W == 128 && c->opt.fuse_small < 2) return 0;   // measured slower than the separate products
  int G, rp;
  leaf_geometry(c, m, &G, &rp);
  if (rp > SN_MAX_RP || small_node_smem(rp, W) > 227 * 1024) return 0;
  r0_for_leaf = r0_for_leaf && W == 64;   // the 128-wide instance does not produce them
  SmallNodeParams p{};
  p.Q1 = Q1;
  p.ldq = ldq;
  p.A2 = A2;
  p.lda = lda;
  p.m = m;
  p.w1 = (int)w1;
  p.w2 = (int)w2;
  p.rows_per_cta = rp;
  p.vec_ok = ((ldq * 2) % 16 == 0) && ((lda * 2) % 16 == 0) && (reinterpret_cast<uintptr_t>(Q1) % 16 == 0) &&
             (reinterpret_cast<uintptr_t>(A2) % 16 == 0);
  p.R12 = R12;
  p.ldr = ldr;
  p.partials = c->d_sn_partials;
  p.r12op = c->d_sn_r12op;
  const size_t mark = c->arena.mark();
  if (W == 128) {   // the opt-in 128-wide instance: its partials come from the arena
    p.partials = static_cast<float*>(c->arena.alloc((size_t)G * 128 * 128 * sizeof(float)));
    if (!p.partials) return 0;   // (no room: the caller runs the separate products)
  }
  p.counter = c->d_counter + 16;
  p.counter_host = &c->counter_host[1];
  p.r0_partials = r0_for_leaf ? c->d_partials : nullptr;
  cudaEvent_t kb = c->kbegin(st);
  cudaError_t e = prec == RGSQR_FP16 ? launch_small_node<__half>(p, G, st) : launch_small_node<__nv_bfloat16>(p, G, st);
  if (e != cudaSuccess) return fail(c, RGSQR_ERR_CUDA, std::string("fused node launch: ") + cudaGetErrorString(e));
  c->kend(3, st, kb, 4.0 * m * w1 * w2, 2.0 * m * (w1 + w2) + 2.0 * m * w2 + 4.0 * w1 * w2);
  c->stats.n_other_launches++;
  c->arena.release(mark);   // (stream-ordered reuse: later kernels on st run after this one)
  return r0_for_leaf ? 2 : 1;
}

// ---------------------------------------------------------------------------------
// in-core recursion (Eq. 2) on a device-resident m x n matrix
// ---------------------------------------------------------------------------------
int64_t split_width(int64_t w, int64_t leaf) {
  if (w <= leaf) return 0;
  int64_t h = (w + 1) / 2;
  int64_t align = w >= 256 ? 64 : 8;
  int64_t w1 = (h + align - 1) / align * align;
  if (w1 >= w) w1 = h;
  return w1;
}

size_t incore_workspace_bytes(Ctx* c, int prec, int64_t m, int64_t n) {
  const int64_t leaf = leaf_width_for(c, m);
  const int64_t w1 = split_width(n, leaf);
  size_t b = 0;
  if (w1 > 0) b += (size_t)w1 * (n - w1) * elem_bytes(prec) + 1024;  // R12 operand copy
  if (w1 > 0 && c->nccl_comm) b += (size_t)w1 * (n - w1) * 4 + 1024;  // R12 rank-reduction buffer
  if (w1 > 0 && c->opt.vshards > 1) b += (size_t)c->opt.vshards * w1 * (n - w1) * 4 + 1024;   // shard partials
  if (prec == RGSQR_TF32X3) b += (size_t)2 * m * n * 4 + 8192;          // hi/lo operands of the top node
  if (c->opt.reorth) {                                                   // CGS2: S (fp32) + leaf S block
    if (w1 > 0) b += (size_t)w1 * (n - w1) * 4 + 1024;
    b += (size_t)LEAF_MAX_W * LEAF_MAX_W * 4 + 1024;
  }
  // split-K partials: op_inner adapts its split factor to what is free; reserve a
  // quarter of the node's matrix bytes, clamped to [1, 16] MiB
  const size_t node_bytes = (size_t)m * n * elem_bytes(prec);
  b += std::min<size_t>((size_t)16 << 20, std::max<size_t>((size_t)1 << 20, node_bytes / 4)) + 4096;
  (void)c;
  return b;
}

struct IncoreCtx {
  Ctx* c;
  int prec;
  char* A;
  int64_t lda, m, s;
  float* R;
  int64_t ldr;
  int64_t leaf;
  void* r12op;
  float* S;        // CGS2: second-pass R12 (fp32, ld w1) of the widest node
  float* S11;      // CGS2: second-pass leaf R block (LEAF_MAX_W x LEAF_MAX_W)
  int64_t col_offset;
  cudaStream_t st;
  IncoreHooks* hooks;
  // deferred products of nodes whose A2 was still being uploaded: R12 = Q1^T A2 and
  // A2 -= Q1 R12 applied chunk by chunk when a descendant first needs the columns
  // (applied in creation order = ancestors first, as the recursion would have)
  bool r0_pre = false;   // the next leaf's round-0 partials were written by the fused node
  struct Deferred {
    int64_t c0, w1, end, applied;
  };
  std::vector<Deferred> deferred;
};

// external projection (ExtProduct) of node columns [applied, upto): chunk by chunk, each
// chunk's upload awaited first
int apply_ext(Ctx* c, int prec, char* A, int64_t lda, int64_t m, IncoreHooks* hk, int64_t upto, cudaStream_t st) {
  ExtProduct* e = hk->ext;
  if (!e) return RGSQR_OK;
  const int64_t s = elem_bytes(prec);
  upto = std::min(upto, e->end);
  const int64_t ch = e->piece > 0 ? e->piece : std::max<int64_t>(hk->chunk, 64);
  while (e->applied < upto) {
    const int64_t a = e->applied, b = std::min(e->end, a + ch);
    hk->need(b);
    const int slot = e->R12[1] ? (e->n_done & 1) : 0;
    if (e->free_ev[slot]) cudaStreamWaitEvent(st, e->free_ev[slot], 0);
    char* A2 = A + a * lda * s;
    int rc = op_inner(c, prec, e->Q1, e->ldq, A2, lda, m, e->w1, b - a, e->R12[slot], e->w1, e->R12op, e->w1, 0, st);
    if (rc < 0) return rc;
    rc = op_outer(c, prec, e->Q1, e->ldq, e->R12op, e->w1, A2, lda, m, e->w1, b - a, st);
    if (rc < 0) return rc;
    e->free_ev[slot] = e->r_out ? e->r_out(a, b, e->R12[slot]) : nullptr;
    e->n_done++;
    e->applied = b;
    if (e->applied >= e->end && e->done) e->done();
  }
  return RGSQR_OK;
}

// columns < col_end: wait for their upload, then apply the deferred products to them
static int incore_need(IncoreCtx& k, int64_t col_end) {
  if (!k.hooks || !k.hooks->need) return RGSQR_OK;
  if (k.hooks->ext) {
    int rc = apply_ext(k.c, k.prec, k.A, k.lda, k.m, k.hooks, col_end, k.st);
    if (rc < 0) return rc;
  }
  for (auto& d : k.deferred) {
    while (d.applied < std::min(col_end, d.end)) {
      // pieces of the upload chunk, or (RGSQR_OPT_DEFER_PIECES = p > 0) about 1/p of the node's A2:
      // narrow pieces let the recursion start on early columns, wide pieces keep the GEMMs efficient
      const int64_t a = d.applied, ch = k.hooks->chunk;
      int64_t piece = ch;
      if (k.c->opt.defer_pieces > 0) {
        const int64_t w2n = d.end - (d.c0 + d.w1);
        piece = std::max(ch, (w2n / k.c->opt.defer_pieces + ch - 1) / ch * ch);
      }
      const int64_t b = piece == ch ? std::min(d.end, (a / ch + 1) * ch) : std::min(d.end, a + piece);
      k.hooks->need(b);
      const int64_t h = d.c0 + d.w1, off = a - h;
      const char* Q1 = k.A + d.c0 * k.lda * k.s;
      char* A2 = k.A + a * k.lda * k.s;
      char* op = static_cast<char*>(k.r12op);
      int rc = op_inner(k.c, k.prec, Q1, k.lda, A2, k.lda, k.m, d.w1, b - a, k.R + d.c0 + a * k.ldr, k.ldr, op,
                        d.w1, 0, k.st);
      if (rc < 0) return rc;
      rc = op_outer(k.c, k.prec, Q1, k.lda, op, d.w1, A2, k.lda, k.m, d.w1, b - a, k.st);
      if (rc < 0) return rc;
      (void)off;
      d.applied = b;
    }
  }
  k.hooks->need(col_end);
  return RGSQR_OK;
}

static int incore_rec(IncoreCtx& k, int64_t c0, int64_t w) {
  const int64_t w1 = split_width(w, k.leaf);
  if (w1 == 0) {
    if (k.hooks && k.hooks->need) {
      int rc = incore_need(k, c0 + w);
      if (rc < 0) return rc;
    }
    char* P = k.A + c0 * k.lda * k.s;
    float* R11 = k.R + c0 + c0 * k.ldr;
    const bool pre = k.r0_pre && !(k.hooks && k.hooks->need && k.hooks->pending && k.hooks->pending(c0 + w));
    int rc = op_leaf(k.c, k.prec, P, k.lda, k.m, w, R11, k.ldr, k.col_offset + c0, k.st, pre);
    if (rc == 0 && k.S11) {
      // CGS2 leaf: factor Q' again, Q' = Q S, and R11 <- S R11
      rc = op_leaf(k.c, k.prec, P, k.lda, k.m, w, k.S11, w, k.col_offset + c0, k.st);
      if (rc == 0) {
        RGSQR_CUDA(k.c, launch_trmm_upper(k.S11, w, R11, k.ldr, (int)w, k.st));
        k.c->stats.n_other_launches++;
      }
    }
    if (rc == 0 && k.hooks && k.hooks->leaf_done) k.hooks->leaf_done(c0 + w);
    return rc;
  }
  const int64_t w2 = w - w1, h = c0 + w1;
  int rc = incore_rec(k, c0, w1);
  if (rc < 0) return rc;
  const char* Q1 = k.A + c0 * k.lda * k.s;
  char* A2 = k.A + h * k.lda * k.s;
  float* R12 = k.R + c0 + h * k.ldr;
  if (k.hooks && k.hooks->pending && k.hooks->chunk > 0 && !k.S && k.hooks->pending(c0 + w)) {
    // A2 is still being uploaded: defer both products; the right child's recursion applies
    // them column chunk by column chunk as it reaches the columns (the columns of
    // R12 = Q1^T A2 and of A2 - Q1 R12 are independent)
    k.deferred.push_back({c0, w1, c0 + w, h});
    k.c->stats.n_incore_nodes++;
    return incore_rec(k, h, w2);
  }
  if (k.hooks && k.hooks->need) {
    rc = incore_need(k, c0 + w);
    if (rc < 0) return rc;
  }
  if (!k.S) {
    // when the right child is a leaf, the fused kernel also hands it its round-0 partials
    const bool right_leaf = split_width(w2, k.leaf) == 0;
    rc = op_small_node(k.c, k.prec, Q1, k.lda, A2, k.lda, k.m, w1, w2, R12, k.ldr, k.st, right_leaf);
    if (rc < 0) return rc;
    if (rc >= 1) {   // done by the fused kernel (2: it also wrote the right leaf's round 0)
      k.c->stats.n_incore_nodes++;
      if (rc == 2) {
        k.r0_pre = true;
        rc = incore_rec(k, h, w2);
        k.r0_pre = false;
        return rc;
      }
      return incore_rec(k, h, w2);
    }
  }
  if (k.prec == RGSQR_TF32X3 && !k.S && !k.c->nccl_comm && k.c->opt.vshards <= 1) {
    rc = op_node_x3(k.c, Q1, k.lda, A2, k.lda, k.m, w1, w2, R12, k.ldr, k.r12op, k.st);
    if (rc < 0) return rc;
  } else {
    rc = op_inner(k.c, k.prec, Q1, k.lda, A2, k.lda, k.m, w1, w2, R12, k.ldr, k.r12op, w1, 0, k.st);
    if (rc < 0) return rc;
    rc = op_outer(k.c, k.prec, Q1, k.lda, k.r12op, w1, A2, k.lda, k.m, w1, w2, k.st);
    if (rc < 0) return rc;
  }
  if (k.S) {
    // CGS2: S = Q1^T A2', A2' -= Q1 S, R12 += S (fixed order)
    rc = op_inner(k.c, k.prec, Q1, k.lda, A2, k.lda, k.m, w1, w2, k.S, w1, k.r12op, w1, 0, k.st);
    if (rc < 0) return rc;
    rc = op_outer(k.c, k.prec, Q1, k.lda, k.r12op, w1, A2, k.lda, k.m, w1, w2, k.st);
    if (rc < 0) return rc;
    cudaError_t e;
    switch (k.prec) {
      case RGSQR_FP16: e = launch_splitk_reduce<__half>(k.S, w1 * w2, w1, 1, R12, k.ldr, 1, nullptr, 0, w1, w2, k.st); break;
      case RGSQR_BF16:
        e = launch_splitk_reduce<__nv_bfloat16>(k.S, w1 * w2, w1, 1, R12, k.ldr, 1, nullptr, 0, w1, w2, k.st);
        break;
      default: e = launch_splitk_reduce<float>(k.S, w1 * w2, w1, 1, R12, k.ldr, 1, nullptr, 0, w1, w2, k.st);
    }
    if (e != cudaSuccess) return fail(k.c, RGSQR_ERR_CUDA, std::string("reorth R12 += S: ") + cudaGetErrorString(e));
    k.c->stats.n_other_launches++;
  }
  k.c->stats.n_incore_nodes++;
  return incore_rec(k, h, w2);
}

int incore_factor(Ctx* c, int prec, void* A, int64_t lda, int64_t m, int64_t n, float* R, int64_t ldr,
                  int64_t col_offset, cudaStream_t st, IncoreHooks* hooks) {
  IncoreCtx k{c, prec, static_cast<char*>(A), lda, m, elem_bytes(prec), R, ldr, leaf_width_for(c, m), nullptr,
              nullptr, nullptr, col_offset, st, hooks};
  if (k.leaf < 1) return fail(c, RGSQR_ERR_UNSUPPORTED, "in-core: m too large for the on-chip leaf");
  const int64_t w1 = split_width(n, k.leaf);
  size_t mark = c->arena.mark();
  if (w1 > 0) {
    k.r12op = c->arena.alloc((size_t)w1 * (n - w1) * k.s);
    if (!k.r12op) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "in-core: no arena space for R12");
    if (c->opt.reorth) {
      k.S = static_cast<float*>(c->arena.alloc((size_t)w1 * (n - w1) * 4));
      if (!k.S) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "in-core: no arena space for the CGS2 R12");
    }
  }
  if (c->opt.reorth) {
    k.S11 = static_cast<float*>(c->arena.alloc((size_t)LEAF_MAX_W * LEAF_MAX_W * 4));
    if (!k.S11) return fail(c, RGSQR_ERR_BUDGET_TOO_SMALL, "in-core: no arena space for the CGS2 leaf block");
  }
  int rc = incore_rec(k, 0, n);
  if (rc >= 0) rc = incore_need(k, n);
  c->arena.release(mark);
  return rc;
}

}  // namespace rgsqr
