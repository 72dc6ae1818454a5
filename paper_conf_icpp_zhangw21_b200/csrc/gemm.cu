// gemm.cu -- the two tensor-core contractions of one recursion node (Eq. 2):
//
//   inner product (TN)  R12 (+)= Q1^T A2      M = w1, N = w2, K = m (rows)
//   outer product (NN)  A2  <-  A2 - Q1 R12   M = m,  N = w2, K = w1
//
// One CTA computes a 128 x BN tile with tcgen05.mma (cta_group::1), operands staged by
// TMA into a STAGES-deep shared-memory ring (128B swizzle), the fp32 accumulator in TMEM.
// Warp roles: warp 0 = TMA producer (one elected lane), warp 1 = MMA issuer (one elected
// lane), warp 2 = TMEM allocator; all four warps run the epilogue (TMEM -> registers ->
// global), warp w owning TMEM lanes [32w, 32w+32).
//
// Column-major storage makes both TN operands K-major (rows are the contraction index);
// in NN the Q1 operand is MN-major (its rows are the output rows) -- legal for
// f16/bf16/tf32 UMMA.  The subtraction A2 - Q1 R12 is fused into the epilogue, so A2'
// is written exactly once, rounded RN-even to the storage type (R5).
#include <algorithm>

#include "dtype.cuh"
#include "kernels.h"
#include "ptx.cuh"

namespace rgsqr {

template <typename T, bool kNN, int BN>
struct GemmCfg {
  static constexpr int BM = 128;
  static constexpr int EPB = 128 / (int)sizeof(T);  // elements per 128-byte row
  static constexpr int BK = EPB;                    // K per pipeline stage
  static constexpr int UK = 32 / (int)sizeof(T);    // K per tcgen05.mma (16 f16, 8 tf32)
  static constexpr int A_BYTES = BM * 128;
  static constexpr int B_BYTES = BN * 128;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int STAGES = (196 * 1024) / STAGE_BYTES > 8 ? 8 : (196 * 1024) / STAGE_BYTES;
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 /*align*/ + 256 /*barriers*/;
  static constexpr uint32_t TMEM_COLS = BN < 32 ? 32 : BN;
  static constexpr uint32_t IDESC = ptx::idesc_f32acc(Elem<T>::kUmmaFormat, kNN ? 1u : 0u, 0u, BM, BN);
};

// Grouped rasterization of a (nx x ny) tile grid launched x-fastest: consecutive CTAs walk GROUP_M
// M-tiles for each N-tile, so a wave of 148 CTAs covers ~16 x 9 tiles and both operands' K-panels are
// re-read from L2 instead of DRAM (the plain x-fastest order re-reads every M-panel once per N-tile:
// 2.5x the algorithmic DRAM bytes at 4096 x 65536 x 4096, profiles/r1_ncu_summary.md)
__device__ __forceinline__ void grouped_tile(int bx, int by, int nx, int ny, int group_m, int* tm, int* tn) {
#ifdef RGSQR_NO_GROUPED_TILE
  *tm = bx;
  *tn = by;
  return;
#endif
  if (group_m <= 1) {
    *tm = bx;
    *tn = by;
    return;
  }
  const int GROUP_M = group_m;
  const int L = by * nx + bx;
  const int per_group = GROUP_M * ny;
  const int g = L / per_group, first = g * GROUP_M;
  const int gsz = min(nx - first, GROUP_M);
  const int r = L - g * per_group;
  *tm = first + r % gsz;
  *tn = r / gsz;
}

template <typename T, bool kNN, int BN>
__global__ void __launch_bounds__(128, 1)
    gemm_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                const __grid_constant__ CUtensorMap mapA2, const __grid_constant__ CUtensorMap mapB2,
                const GemmParams p, const int group_m) {
  using C = GemmCfg<T, kNN, BN>;
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = ptx::smem_u32(smem_raw);
  uint8_t* smem = smem_raw + (((raw + 1023u) & ~1023u) - raw);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + C::STAGES * C::STAGE_BYTES);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tfull = empty + C::STAGES;
  uint32_t* tslot = reinterpret_cast<uint32_t*>(tfull + 1);

  const int warp = threadIdx.x >> 5;
  int tm, tn;
  grouped_tile(blockIdx.x, blockIdx.y, gridDim.x, gridDim.y, group_m, &tm, &tn);
  const int64_t m0 = (int64_t)tm * C::BM;
  const int64_t n0 = (int64_t)tn * BN;
  const int64_t kb0 = (int64_t)blockIdx.z * p.kb_per_split;
  const int64_t kb1 = min(p.kb_total, kb0 + p.kb_per_split);
  const int nkb = (int)(kb1 - kb0);

  if (warp == 0 && ptx::elect_one()) {
    ptx::tma_prefetch_desc(&mapA);
    ptx::tma_prefetch_desc(&mapB);
    if (p.kb_seg > 0) {
      ptx::tma_prefetch_desc(&mapA2);
      ptx::tma_prefetch_desc(&mapB2);
    }
    for (int s = 0; s < C::STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    ptx::mbar_init(tfull, 1);
    ptx::fence_mbar_init();
  }
  if (warp == 2) ptx::tmem_alloc<C::TMEM_COLS>(tslot);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tslot;

  if (warp == 0) {
    // ---------------- TMA producer ----------------
    if (ptx::elect_one()) {
      for (int it = 0; it < nkb; ++it) {
        const int s = it % C::STAGES;
        const uint32_t ph = (uint32_t)(it / C::STAGES) & 1u;
        ptx::mbar_wait(&empty[s], ph ^ 1u);
        uint8_t* sA = smem + s * C::STAGE_BYTES;
        uint8_t* sB = sA + C::A_BYTES;
        // TF32X3 segments (p.kb_seg > 0): k-blocks [0, kb_seg) = (A, B lo), then (A lo, B), then
        // (A, B): the small cross terms accumulate first -- the tensor core's fp32 accumulation
        // aligns to the largest addend, so adding them after the big term would drop their low bits
        int64_t kbg = kb0 + it;
        int seg = 2;
        if (p.kb_seg > 0) {
          seg = (int)(kbg / p.kb_seg);
          kbg -= (int64_t)seg * p.kb_seg;
        }
        const CUtensorMap* ta = seg == 1 ? &mapA2 : &mapA;
        const CUtensorMap* tb = seg == 0 ? &mapB2 : &mapB;
        const int32_t k0 = (int32_t)(kbg * C::BK);
        ptx::mbar_arrive_expect_tx(&full[s], C::STAGE_BYTES);
        if constexpr (kNN) {
#pragma unroll
          for (int mb = 0; mb < C::BM / C::EPB; ++mb)
            ptx::tma_load_2d(sA + mb * C::BK * 128, ta, &full[s], (int32_t)(m0 + mb * C::EPB), k0);
        } else {
          ptx::tma_load_2d(sA, ta, &full[s], k0, (int32_t)m0);
        }
        ptx::tma_load_2d(sB, tb, &full[s], k0, (int32_t)n0);
      }
    }
  } else if (warp == 1) {
    // ---------------- MMA issuer ----------------
    if (ptx::elect_one()) {
      for (int it = 0; it < nkb; ++it) {
        const int s = it % C::STAGES;
        const uint32_t ph = (uint32_t)(it / C::STAGES) & 1u;
        ptx::mbar_wait(&full[s], ph);
        ptx::tc_fence_after();
        const uint32_t aBase = ptx::smem_u32(smem + s * C::STAGE_BYTES);
        const uint32_t bBase = aBase + C::A_BYTES;
#pragma unroll
        for (int kk = 0; kk < C::BK / C::UK; ++kk) {
          uint64_t ad;
          if constexpr (kNN && Elem<T>::kTF32)
            ad = ptx::sdesc_sw128(aBase + kk * C::UK * 128, C::BK * 128, 512, 1);
          else if constexpr (kNN)
            ad = ptx::sdesc_sw128(aBase + kk * C::UK * 128, C::BK * 128, 1024);
          else
            ad = ptx::sdesc_sw128(aBase + kk * C::UK * (int)sizeof(T), 16, 1024);
          const uint64_t bd = ptx::sdesc_sw128(bBase + kk * C::UK * (int)sizeof(T), 16, 1024);
          ptx::umma<Elem<T>::kTF32>(tmem, ad, bd, C::IDESC, (it | kk) != 0 ? 1u : 0u);
        }
        ptx::umma_commit(&empty[s]);
      }
      ptx::umma_commit(tfull);
    }
  }
  __syncwarp();

  // ---------------- epilogue: all four warps ----------------
  // Thread (warp w, lane l) owns output row i = m0 + 32w + l; per 32-column chunk it
  // reads its TMEM lane, and (NN / accumulating TN) the old values of its row, which
  // are loaded one chunk ahead with predicated, branch-free loads so that the 32 loads
  // of a chunk are in flight together (the first chunk before the accumulator is ready).
  const int lane = threadIdx.x & 31;
  const int64_t i = m0 + warp * 32 + lane;
  const bool row_ok = i < p.M;
  const bool needs_old = kNN || (p.P == nullptr && p.accumulate);
  float old[32], nxt[32];
  auto load_chunk = [&](int cc, float (&dst)[32]) {
    const int64_t nb = n0 + cc * 32;
#pragma unroll
    for (int j = 0; j < 32; ++j) {
      const int64_t n = nb + j;
      const bool ok = row_ok && n < p.N;
      if constexpr (kNN)
        dst[j] = ok ? Elem<T>::load(__ldcs(reinterpret_cast<const T*>(p.A2) + i + n * p.lda2)) : 0.0f;
      else
        dst[j] = ok ? __ldcs(p.C + i + n * p.ldc) : 0.0f;
    }
  };
  if (needs_old) load_chunk(0, old);
  if (nkb > 0) ptx::mbar_wait(tfull, 0);
  ptx::tc_fence_after();
#pragma unroll 1
  for (int cc = 0; cc < BN / 32; ++cc) {
    if (n0 + cc * 32 >= p.N) break;  // warp-uniform
    if (needs_old && cc + 1 < BN / 32) load_chunk(cc + 1, nxt);
    uint32_t v[32];
    if (nkb > 0) {
      ptx::tmem_ld_32x32b_x32(tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)(cc * 32), v);
      ptx::tmem_ld_wait();
    } else {
#pragma unroll
      for (int j = 0; j < 32; ++j) v[j] = 0u;
    }
    const int64_t nb = n0 + cc * 32;
#pragma unroll
    for (int j = 0; j < 32; ++j) {
      const int64_t n = nb + j;
      const bool ok = row_ok && n < p.N;
      const float x = __uint_as_float(v[j]);
      if constexpr (kNN) {
        if (ok) reinterpret_cast<T*>(p.A2)[i + n * p.lda2] = Elem<T>::store(old[j] - x);
      } else {
        if (p.P != nullptr) {
          if (ok) p.P[blockIdx.z * p.split_stride + i + n * p.ldp] = x;
        } else {
          const float y = p.accumulate ? old[j] + x : x;
          if (ok) p.C[i + n * p.ldc] = y;
          if (ok && p.Cop != nullptr) reinterpret_cast<T*>(p.Cop)[i + n * p.ldop] = Elem<T>::store(y);
        }
      }
    }
    if (needs_old) {
#pragma unroll
      for (int j = 0; j < 32; ++j) old[j] = nxt[j];
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<C::TMEM_COLS>(tmem);
  }
}

// ---------------------------------------------------------------------------------
// Inner product with a bounded tensor-core accumulation chain (TF32X3, fp32 operands;
// DESIGN.md R25).  The tcgen05 fp32 accumulation drops low bits at every add, so its error grows
// linearly with the number of k-blocks summed in TMEM (measured: ~1.5e-7 relative per k-block,
// profiles/r2_x3_chain_before_promotion.json).  Here the MMA warp accumulates units of
// p.kb_per_unit k-blocks into one of TWO TMEM accumulators, and the epilogue warps fold every unit
// into fp32 registers (round-to-nearest adds) while the next unit is being accumulated.
// Warp roles (256 threads): 0 TMA, 1 MMA, 2 TMEM allocator, 4..7 accumulate + epilogue (warp w
// owns TMEM lanes [32 (w-4), 32 (w-4) + 32)).  Output as gemm_kernel's TN epilogue.
// ---------------------------------------------------------------------------------
template <int BN>
__global__ void __launch_bounds__(128 + 16 * 32, 1)
    tn_promote_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                      const __grid_constant__ CUtensorMap mapA2, const __grid_constant__ CUtensorMap mapB2,
                      const GemmParams p, const GemmExtra x) {
  using C = GemmCfg<float, false, BN>;
  static_assert(2 * BN <= 512, "two accumulators must fit TMEM");
  static_assert(BN == 128, "16 accumulation warps x 32 columns");
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = ptx::smem_u32(smem_raw);
  uint8_t* smem = smem_raw + (((raw + 1023u) & ~1023u) - raw);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + C::STAGES * C::STAGE_BYTES);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tfull = empty + C::STAGES;   // [2]
  uint64_t* tempty = tfull + 2;          // [2]
  uint32_t* tslot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5;
  int tm, tn;
  grouped_tile(blockIdx.x, blockIdx.y, gridDim.x, gridDim.y, x.group_m, &tm, &tn);
  const int64_t m0 = (int64_t)tm * C::BM;
  const int64_t n0 = (int64_t)tn * BN;
  const int64_t kb0 = (int64_t)blockIdx.z * p.kb_per_split;
  const int64_t kb1 = min(p.kb_total, kb0 + p.kb_per_split);
  const int nkb = kb1 > kb0 ? (int)(kb1 - kb0) : 0;
  const int pk = x.kb_per_unit > 0 ? (int)x.kb_per_unit : max(nkb, 1);
  const int nunits = nkb > 0 ? (nkb + pk - 1) / pk : 0;

  if (warp == 0 && ptx::elect_one()) {
    ptx::tma_prefetch_desc(&mapA);
    ptx::tma_prefetch_desc(&mapB);
    ptx::tma_prefetch_desc(&mapA2);
    ptx::tma_prefetch_desc(&mapB2);
    for (int s = 0; s < C::STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      ptx::mbar_init(&tfull[b], 1);
      ptx::mbar_init(&tempty[b], 16);
    }
    ptx::fence_mbar_init();
  }
  if (warp == 2) ptx::tmem_alloc<2 * BN>(tslot);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tslot;

  if (warp == 0) {
    if (ptx::elect_one()) {
      for (int it = 0; it < nkb; ++it) {
        const int s = it % C::STAGES;
        const uint32_t ph = (uint32_t)(it / C::STAGES) & 1u;
        ptx::mbar_wait(&empty[s], ph ^ 1u);
        uint8_t* sA = smem + s * C::STAGE_BYTES;
        uint8_t* sB = sA + C::A_BYTES;
        int64_t kbg = kb0 + it;
        int seg = 2;
        if (p.kb_seg > 0) {
          seg = (int)(kbg / p.kb_seg);
          kbg -= (int64_t)seg * p.kb_seg;
        }
        const CUtensorMap* ta = seg == 1 ? &mapA2 : &mapA;
        const CUtensorMap* tb = seg == 0 ? &mapB2 : &mapB;
        const int32_t k0 = (int32_t)(kbg * C::BK);
        ptx::mbar_arrive_expect_tx(&full[s], C::STAGE_BYTES);
        ptx::tma_load_2d(sA, ta, &full[s], k0, (int32_t)m0);
        ptx::tma_load_2d(sB, tb, &full[s], k0, (int32_t)n0);
      }
    }
  } else if (warp == 1) {
    if (ptx::elect_one()) {
      int it = 0;
      for (int u = 0; u < nunits; ++u) {
        const int b = u & 1;
        ptx::mbar_wait(&tempty[b], ((uint32_t)(u >> 1) & 1u) ^ 1u);
        ptx::tc_fence_after();
        const uint32_t acc = tmem + (uint32_t)(b * BN);
        const int q1 = min(nkb, (u + 1) * pk);
        for (; it < q1; ++it) {
          const int s = it % C::STAGES;
          ptx::mbar_wait(&full[s], (uint32_t)(it / C::STAGES) & 1u);
          ptx::tc_fence_after();
          const uint32_t aBase = ptx::smem_u32(smem + s * C::STAGE_BYTES);
          const uint32_t bBase = aBase + C::A_BYTES;
#pragma unroll
          for (int kk = 0; kk < C::BK / C::UK; ++kk) {
            const uint64_t ad = ptx::sdesc_sw128(aBase + kk * C::UK * 4, 16, 1024);
            const uint64_t bd = ptx::sdesc_sw128(bBase + kk * C::UK * 4, 16, 1024);
            ptx::umma<true>(acc, ad, bd, C::IDESC, (it != u * pk || kk != 0) ? 1u : 0u);
          }
          ptx::umma_commit(&empty[s]);
        }
        ptx::umma_commit(&tfull[b]);
      }
    }
  } else if (warp >= 4) {
    // 16 accumulation warps: warp w reads TMEM lanes [32 (w % 4), +32) (its lane quadrant) and
    // columns [32 cg, 32 cg + 32), cg = (w - 4) / 4.  The unit sums accumulate in fp64: with K = m
    // there can be thousands of units, and an fp32 running sum would add a random-walk error of
    // sqrt(units) * 2^-24 (R25)
    const int q = warp & 3, cg = (warp - 4) >> 2, lane = threadIdx.x & 31;
    double sum[32];
#pragma unroll
    for (int j = 0; j < 32; ++j) sum[j] = 0.0;
    for (int u = 0; u < nunits; ++u) {
      const int b = u & 1;
      ptx::mbar_wait(&tfull[b], (uint32_t)(u >> 1) & 1u);
      ptx::tc_fence_after();
#pragma unroll
      for (int h = 0; h < 2; ++h) {   // two 16-column loads (register pressure at 640 threads)
        uint32_t v[16];
        ptx::tmem_ld_32x32b_x16(tmem + (uint32_t)(b * BN) + ((uint32_t)(q * 32) << 16) + (uint32_t)(cg * 32 + h * 16), v);
        ptx::tmem_ld_wait();
#pragma unroll
        for (int j = 0; j < 16; ++j) sum[h * 16 + j] += (double)__uint_as_float(v[j]);
      }
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&tempty[b]);
    }
    const int64_t i = m0 + q * 32 + lane;
    if (i < p.M) {
#pragma unroll
      for (int j = 0; j < 32; ++j) {
        const int64_t n = n0 + cg * 32 + j;
        if (n < p.N) {
          if (p.P != nullptr) {
            p.P[blockIdx.z * p.split_stride + i + n * p.ldp] = (float)sum[j];
          } else {
            const float y = p.accumulate ? (float)((double)p.C[i + n * p.ldc] + sum[j]) : (float)sum[j];
            p.C[i + n * p.ldc] = y;
            if (p.Cop != nullptr) reinterpret_cast<float*>(p.Cop)[i + n * p.ldop] = y;
          }
        }
      }
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<2 * BN>(tmem);
  }
}

// ---------------------------------------------------------------------------------
// Deterministic split-K reduction: C = (accumulate ? C : 0) + sum_{s=0..S-1} P[s] in
// a fixed order (no float atomics; R10), plus the optional operand copy.
// ---------------------------------------------------------------------------------
template <typename T>
__global__ void splitk_reduce_kernel(const float* __restrict__ P, int64_t split_stride, int64_t ldp,
                                     int splits, float* C, int64_t ldc, int accumulate, T* Cop,
                                     int64_t ldop, int64_t M, int64_t N) {
  const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= M * N) return;
  const int64_t i = idx % M, n = idx / M;
  float acc = accumulate ? C[i + n * ldc] : 0.0f;
  for (int s = 0; s < splits; ++s) acc += P[s * split_stride + i + n * ldp];
  C[i + n * ldc] = acc;
  if (Cop != nullptr) Cop[i + n * ldop] = Elem<T>::store(acc);
}

// ---------------------------------------------------------------------------------
// Persistent outer-product kernel  A2 <- A2 - Q1 R12.
//
// One CTA per SM loops over 128 x BN output tiles (tile = tm * tiles_n + tn, so
// consecutive tiles of a CTA share Q1 rows in L2).  Warp roles (256 threads):
//   warp 0      TMA producer of the Q1 / R12 k-blocks (STAGES-deep ring)
//   warp 1      MMA issuer (tcgen05.mma, fp32 accumulator in TMEM, TWO accumulator
//               buffers so the epilogue of tile j overlaps the MMAs of tile j+1)
//   warp 2      TMEM allocator + TMA loader of the OLD A2 tile into a shared-memory C tile
//   warps 4..7  epilogue: TMEM -> registers, C = C - acc in shared memory, rounded RN to
//               the storage type, TMA store of the tile (one write of A2' per element)
// ---------------------------------------------------------------------------------
template <typename T, int BN>
struct NNCfg {
  static constexpr int BM = 128;
  static constexpr int EPB = 128 / (int)sizeof(T);
  static constexpr int BK = EPB;
  static constexpr int UK = 32 / (int)sizeof(T);
  static constexpr int A_BYTES = BM * 128;
  static constexpr int B_BYTES = BN * 128;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int CBOX_N = 64;                                 // columns per C TMA box
  static constexpr int C_BYTES = BM * BN * (int)sizeof(T);
  // two C tiles (the old-A2 load of tile j+1 overlaps the epilogue of tile j) when at least
  // three k-stages still fit; otherwise one
  static constexpr int STAGES2 = (220 * 1024 - 2 * C_BYTES - 2048) / STAGE_BYTES;
  static constexpr int C_BUFS = STAGES2 >= 3 ? 2 : 1;
  static constexpr int STAGES_RAW = (220 * 1024 - C_BUFS * C_BYTES - 2048) / STAGE_BYTES;
  static constexpr int STAGES = STAGES_RAW > 8 ? 8 : STAGES_RAW;
  static constexpr int SMEM = STAGES * STAGE_BYTES + C_BUFS * C_BYTES + 1024 + 512;
  static constexpr uint32_t TMEM_COLS = 2 * BN < 32 ? 32 : 2 * BN;
  static constexpr uint32_t IDESC = ptx::idesc_f32acc(Elem<T>::kUmmaFormat, 1u, 0u, BM, BN);
  static_assert(STAGES >= 2, "NN tile does not fit shared memory");
  static_assert(2 * BN <= 512, "two accumulators must fit TMEM");
};

template <typename T, int BN>
__global__ void __launch_bounds__(256, 1)
    nn_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
              const __grid_constant__ CUtensorMap mapC, const __grid_constant__ CUtensorMap mapA2,
              const __grid_constant__ CUtensorMap mapB2, const NNParams p) {
  using C = NNCfg<T, BN>;
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = ptx::smem_u32(smem_raw);
  uint8_t* smem = smem_raw + (((raw + 1023u) & ~1023u) - raw);
  T* Cs0 = reinterpret_cast<T*>(smem + C::STAGES * C::STAGE_BYTES);   // [C_BUFS] C tiles
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + C::STAGES * C::STAGE_BYTES + C::C_BUFS * C::C_BYTES);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tfull = empty + C::STAGES;   // [2]
  uint64_t* tempty = tfull + 2;          // [2]
  uint64_t* cfull = tempty + 2;          // [C_BUFS]
  uint64_t* cempty = cfull + C::C_BUFS;  // [C_BUFS]
  uint32_t* tslot = reinterpret_cast<uint32_t*>(cempty + C::C_BUFS);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int num_tiles = p.tiles_m * p.tiles_n;
  const int nkb = (int)p.kb_total;
  const int pk = p.promote_kb > 0 ? (int)p.promote_kb : max(nkb, 1);   // k-blocks per accumulation unit

  if (warp == 0 && ptx::elect_one()) {
    ptx::tma_prefetch_desc(&mapA);
    ptx::tma_prefetch_desc(&mapB);
    ptx::tma_prefetch_desc(&mapC);
    for (int s = 0; s < C::STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      ptx::mbar_init(&tfull[b], 1);
      ptx::mbar_init(&tempty[b], 4);
    }
    for (int b = 0; b < C::C_BUFS; ++b) {
      ptx::mbar_init(&cfull[b], 1);
      ptx::mbar_init(&cempty[b], 1);
    }
    ptx::fence_mbar_init();
  }
  if (warp == 2) ptx::tmem_alloc<C::TMEM_COLS>(tslot);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tslot;

  if (warp == 0) {
    if (ptx::elect_one()) {
      int it = 0;
      for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x) {
        const int32_t m0 = (tile / p.tiles_n) * C::BM, n0 = (tile % p.tiles_n) * BN;
        for (int kb = 0; kb < nkb; ++kb, ++it) {
          const int s = it % C::STAGES;
          ptx::mbar_wait(&empty[s], ((uint32_t)(it / C::STAGES) & 1u) ^ 1u);
          uint8_t* sA = smem + s * C::STAGE_BYTES;
          // TF32X3 segments (p.kb_seg > 0): (A, B lo), (A lo, B), then (A, B) -- small terms first
          int seg = 2, kbl = kb;
          if (p.kb_seg > 0) {
            seg = kb / (int)p.kb_seg;
            kbl = kb - seg * (int)p.kb_seg;
          }
          const CUtensorMap* ta = seg == 1 ? &mapA2 : &mapA;
          const CUtensorMap* tb = seg == 0 ? &mapB2 : &mapB;
          const int32_t k0 = kbl * C::BK;
          ptx::mbar_arrive_expect_tx(&full[s], C::STAGE_BYTES);
#pragma unroll
          for (int mb = 0; mb < C::BM / C::EPB; ++mb)
            ptx::tma_load_2d(sA + mb * C::BK * 128, ta, &full[s], m0 + mb * C::EPB, k0);
          ptx::tma_load_2d(sA + C::A_BYTES, tb, &full[s], k0, n0);
        }
      }
    }
  } else if (warp == 1) {
    if (ptx::elect_one()) {
      // accumulation units: a tile's K range in chains of `pk` k-blocks (p.promote_kb; the whole K
      // when 0), alternating between the two TMEM accumulators; the epilogue folds each unit into
      // the fp32 C tile in shared memory (RN), bounding the tensor core's accumulation chain
      int it = 0, u = 0;
      for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x) {
        for (int q0 = 0; q0 < nkb || q0 == 0; q0 += pk, ++u) {
          const int b = u & 1;
          ptx::mbar_wait(&tempty[b], ((uint32_t)(u >> 1) & 1u) ^ 1u);
          ptx::tc_fence_after();
          const uint32_t acc = tmem + (uint32_t)(b * BN);
          const int q1 = min(nkb, q0 + pk);
          for (int kb = q0; kb < q1; ++kb, ++it) {
            const int s = it % C::STAGES;
            ptx::mbar_wait(&full[s], (uint32_t)(it / C::STAGES) & 1u);
            ptx::tc_fence_after();
            const uint32_t aBase = ptx::smem_u32(smem + s * C::STAGE_BYTES);
            const uint32_t bBase = aBase + C::A_BYTES;
#pragma unroll
            for (int kk = 0; kk < C::BK / C::UK; ++kk) {
              uint64_t ad;
              if constexpr (Elem<T>::kTF32)
                ad = ptx::sdesc_sw128(aBase + kk * C::UK * 128, C::BK * 128, 512, 1);
              else
                ad = ptx::sdesc_sw128(aBase + kk * C::UK * 128, C::BK * 128, 1024);
              const uint64_t bd = ptx::sdesc_sw128(bBase + kk * C::UK * (int)sizeof(T), 16, 1024);
              ptx::umma<Elem<T>::kTF32>(acc, ad, bd, C::IDESC, (kb != q0 || kk != 0) ? 1u : 0u);
            }
            ptx::umma_commit(&empty[s]);
          }
          ptx::umma_commit(&tfull[b]);
          if (nkb == 0) break;
        }
      }
    }
  } else if (warp == 2) {
    if (ptx::elect_one()) {
      int lt = 0;
      for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x, ++lt) {
        const int32_t m0 = (tile / p.tiles_n) * C::BM, n0 = (tile % p.tiles_n) * BN;
        const int cbuf = lt % C::C_BUFS;
        const uint32_t cph = (uint32_t)(lt / C::C_BUFS) & 1u;
        T* Cs = Cs0 + cbuf * (C::C_BYTES / (int)sizeof(T));
        ptx::mbar_wait(&cempty[cbuf], cph ^ 1u);
        ptx::mbar_arrive_expect_tx(&cfull[cbuf], C::C_BYTES);
#pragma unroll
        for (int cb = 0; cb < BN / C::CBOX_N; ++cb)
          ptx::tma_load_2d(Cs + cb * C::CBOX_N * C::BM, &mapC, &cfull[cbuf], m0, n0 + cb * C::CBOX_N);
      }
    }
  } else if (warp >= 4) {
    const int ew = warp - 4;                 // == warp % 4: TMEM lanes [32 ew, 32 ew + 32)
    const int r = ew * 32 + lane;            // row within the tile
    int lt = 0, u = 0;
    for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x, ++lt) {
      const int32_t m0 = (tile / p.tiles_n) * C::BM, n0 = (tile % p.tiles_n) * BN;
      const int cbuf = lt % C::C_BUFS;
      T* Cs = Cs0 + cbuf * (C::C_BYTES / (int)sizeof(T));
      ptx::mbar_wait(&cfull[cbuf], (uint32_t)(lt / C::C_BUFS) & 1u);
      for (int q0 = 0; q0 < nkb || q0 == 0; q0 += pk, ++u) {
        const int b = u & 1;
        ptx::mbar_wait(&tfull[b], (uint32_t)(u >> 1) & 1u);
        ptx::tc_fence_after();
#pragma unroll 1
        for (int cc = 0; cc < BN / 32; ++cc) {
          uint32_t v[32];
          ptx::tmem_ld_32x32b_x32(tmem + (uint32_t)(b * BN) + ((uint32_t)(ew * 32) << 16) + (uint32_t)(cc * 32), v);
          ptx::tmem_ld_wait();
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            T* cp = Cs + (cc * 32 + j) * C::BM + r;
            *cp = Elem<T>::store(Elem<T>::load(*cp) - __uint_as_float(v[j]));
          }
        }
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(&tempty[b]);
        if (nkb == 0) break;
      }
      ptx::fence_proxy_async();              // generic smem writes -> visible to the TMA store
      ptx::named_bar_sync(1, 128);
      if (ew == 0 && lane == 0) {
#pragma unroll
        for (int cb = 0; cb < BN / C::CBOX_N; ++cb)
          ptx::tma_store_2d(&mapC, Cs + cb * C::CBOX_N * C::BM, m0, n0 + cb * C::CBOX_N);
        ptx::bulk_commit();
        ptx::bulk_wait_read0();
        ptx::mbar_arrive(&cempty[cbuf]);
      }
    }
    if (ew == 0 && lane == 0) ptx::bulk_wait0();
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<C::TMEM_COLS>(tmem);
  }
}

template <typename T, int BN>
static cudaError_t launch_nn_t(const CUtensorMap& ma, const CUtensorMap& mb, const CUtensorMap& mc,
                               const CUtensorMap& ma2, const CUtensorMap& mb2, const NNParams& p, int grid,
                               cudaStream_t st) {
  using C = NNCfg<T, BN>;
  static bool attr_set = false;
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(nn_kernel<T, BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  nn_kernel<T, BN><<<grid, 256, C::SMEM, st>>>(ma, mb, mc, ma2, mb2, p);
  return cudaGetLastError();
}

template <typename T>
cudaError_t launch_nn(int bn, const CUtensorMap& ma, const CUtensorMap& mb, const CUtensorMap& mc,
                      const NNParams& p, int grid, cudaStream_t st, const CUtensorMap* ma2, const CUtensorMap* mb2) {
  const CUtensorMap& a2 = ma2 ? *ma2 : ma;
  const CUtensorMap& b2 = mb2 ? *mb2 : mb;
  if constexpr (sizeof(T) == 4) {
    if (bn >= 128) return launch_nn_t<T, 128>(ma, mb, mc, a2, b2, p, grid, st);
    return launch_nn_t<T, 64>(ma, mb, mc, a2, b2, p, grid, st);
  } else {
    if (bn == 256) return launch_nn_t<T, 256>(ma, mb, mc, a2, b2, p, grid, st);
    if (bn == 128) return launch_nn_t<T, 128>(ma, mb, mc, a2, b2, p, grid, st);
    return launch_nn_t<T, 64>(ma, mb, mc, a2, b2, p, grid, st);
  }
}

template cudaError_t launch_nn<__half>(int, const CUtensorMap&, const CUtensorMap&, const CUtensorMap&, const NNParams&,
                                int, cudaStream_t, const CUtensorMap*, const CUtensorMap*);
template cudaError_t launch_nn<__nv_bfloat16>(int, const CUtensorMap&, const CUtensorMap&, const CUtensorMap&, const NNParams&,
                                int, cudaStream_t, const CUtensorMap*, const CUtensorMap*);
template cudaError_t launch_nn<float>(int, const CUtensorMap&, const CUtensorMap&, const CUtensorMap&, const NNParams&,
                                int, cudaStream_t, const CUtensorMap*, const CUtensorMap*);

// ---------------------------------------------------------------------------------
// host-side launch helpers
// ---------------------------------------------------------------------------------
template <typename T, bool kNN, int BN>
static cudaError_t launch_gemm_t(const CUtensorMap& ma, const CUtensorMap& mb, const CUtensorMap& ma2,
                                 const CUtensorMap& mb2, const GemmParams& p, int splits, cudaStream_t st,
                                 int group_m) {
  using C = GemmCfg<T, kNN, BN>;
  static bool attr_set = false;
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(gemm_kernel<T, kNN, BN>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  dim3 grid((unsigned)((p.M + C::BM - 1) / C::BM), (unsigned)((p.N + BN - 1) / BN), (unsigned)splits);
  gemm_kernel<T, kNN, BN><<<grid, 128, C::SMEM, st>>>(ma, mb, ma2, mb2, p, group_m);
  return cudaGetLastError();
}

template <int BN>
static cudaError_t launch_tn_promote_t(const CUtensorMap& ma, const CUtensorMap& mb, const CUtensorMap& ma2,
                                       const CUtensorMap& mb2, const GemmParams& p, int splits, cudaStream_t st,
                                       const GemmExtra& x) {
  using C = GemmCfg<float, false, BN>;
  constexpr int SMEM = C::SMEM + 64;
  static bool attr_set = false;
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(tn_promote_kernel<BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  dim3 grid((unsigned)((p.M + C::BM - 1) / C::BM), (unsigned)((p.N + BN - 1) / BN), (unsigned)splits);
  tn_promote_kernel<BN><<<grid, 128 + 16 * 32, SMEM, st>>>(ma, mb, ma2, mb2, p, x);
  return cudaGetLastError();
}

template <typename T>
cudaError_t launch_gemm(bool nn, int bn, const CUtensorMap& ma, const CUtensorMap& mb,
                        const GemmParams& p, int splits, cudaStream_t st, const CUtensorMap* ma2,
                        const CUtensorMap* mb2, GemmExtra x) {
  const CUtensorMap& a2 = ma2 ? *ma2 : ma;
  const CUtensorMap& b2 = mb2 ? *mb2 : mb;
  if constexpr (sizeof(T) == 4) {
    if (!nn && x.kb_per_unit > 0)   // bounded accumulation chain (TF32X3), fp64 unit sums
      return launch_tn_promote_t<128>(ma, mb, a2, b2, p, splits, st, x);
  }
  const int g = x.group_m;
  if (nn) {
    if (bn == 256) return launch_gemm_t<T, true, 256>(ma, mb, a2, b2, p, splits, st, g);
    if (bn == 128) return launch_gemm_t<T, true, 128>(ma, mb, a2, b2, p, splits, st, g);
    return launch_gemm_t<T, true, 64>(ma, mb, a2, b2, p, splits, st, g);
  }
  if (bn == 256) return launch_gemm_t<T, false, 256>(ma, mb, a2, b2, p, splits, st, g);
  if (bn == 128) return launch_gemm_t<T, false, 128>(ma, mb, a2, b2, p, splits, st, g);
  return launch_gemm_t<T, false, 64>(ma, mb, a2, b2, p, splits, st, g);
}

// Many splits: a CTA owns 32 consecutive output elements (coalesced 128-byte reads of every
// split's partial); its 8 warps each sum every 8th split (two interleaved chains), then warp 0
// adds the 8 group sums -- a fixed order, so the result is deterministic.
template <typename T>
__global__ void __launch_bounds__(256) splitk_reduce_group_kernel(const float* __restrict__ P, int64_t split_stride,
                                                                  int64_t ldp, int splits, float* C, int64_t ldc,
                                                                  int accumulate, T* Cop, int64_t ldop, int64_t M,
                                                                  int64_t N) {
  __shared__ float red[8][33];
  const int o = threadIdx.x & 31, g = threadIdx.x >> 5;
  const int64_t idx = (int64_t)blockIdx.x * 32 + o;
  const bool ok = idx < M * N;
  const int64_t i = ok ? idx % M : 0, n = ok ? idx / M : 0;
  const float* base = P + i + n * ldp;
  float a0 = 0.f, a1 = 0.f;
  if (ok) {
    int s = g;
    // Four iterations of the pair loop below with their 8 loads issued together (the reduce is
    // latency-bound at small M N); summation order unchanged, so results are bitwise the same.
    // (A 16-load version with predicated tail loads was slower: 27.7 vs 13.8 us at M = N = 512.)
    for (; s + 56 < splits; s += 64) {
      float v[8];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        v[2 * u] = __ldcs(base + (s + 16 * u) * split_stride);
        v[2 * u + 1] = __ldcs(base + (s + 16 * u + 8) * split_stride);
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        a0 += v[2 * u];
        a1 += v[2 * u + 1];
      }
    }
    for (; s + 8 < splits; s += 16) {
      a0 += __ldcs(base + s * split_stride);
      a1 += __ldcs(base + (s + 8) * split_stride);
    }
    if (s < splits) a0 += __ldcs(base + s * split_stride);
  }
  red[g][o] = a0 + a1;
  __syncthreads();
  if (g == 0 && ok) {
    float acc = red[0][o];
#pragma unroll
    for (int q = 1; q < 8; ++q) acc += red[q][o];
    if (accumulate) acc = C[i + n * ldc] + acc;
    C[i + n * ldc] = acc;
    if (Cop != nullptr) Cop[i + n * ldop] = Elem<T>::store(acc);
  }
}

template <typename T>
cudaError_t launch_splitk_reduce(const float* P, int64_t split_stride, int64_t ldp, int splits,
                                 float* C, int64_t ldc, int accumulate, T* Cop, int64_t ldop,
                                 int64_t M, int64_t N, cudaStream_t st) {
  const int64_t total = M * N;
  const int threads = 256;
  if (splits >= 8) {
    splitk_reduce_group_kernel<T><<<(unsigned)((total + 31) / 32), 256, 0, st>>>(
        P, split_stride, ldp, splits, C, ldc, accumulate, Cop, ldop, M, N);
  } else {
    splitk_reduce_kernel<T><<<(unsigned)((total + threads - 1) / threads), threads, 0, st>>>(
        P, split_stride, ldp, splits, C, ldc, accumulate, Cop, ldop, M, N);
  }
  return cudaGetLastError();
}

int gemm_block_k(int elem_bytes) { return 128 / elem_bytes; }

// TF32X3 operand split (R25): hi = RN_tf32(x), lo = RN_tf32(x - hi),
// both written as fp32 words whose low 13 mantissa bits are zero, so tcgen05 kind::tf32 (which
// reads the top 19 bits) consumes them exactly.  |x - hi - lo| <= 2^-22 |x| and the dropped
// lo*lo term is <= 2^-22 |x||y| (truncated parts would give 2^-20 for both).  x - hi is exact in
// fp32.  RN-even by integer rounding of the bit pattern (finite inputs).
__device__ __forceinline__ float rn_tf32(float x) {
  const uint32_t u = __float_as_uint(x);
  return __uint_as_float((u + 0xFFFu + ((u >> 13) & 1u)) & 0xFFFFE000u);
}

__global__ void tf32_split_kernel(const float* __restrict__ src, int64_t lds, float* __restrict__ hi, int64_t ldh,
                                  float* __restrict__ lo, int64_t ldl, int64_t M, int64_t N, int vec) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  if (vec) {   // M, lds, ldh, ldl multiples of 4, 16-byte aligned bases
    const int64_t M4 = M / 4, total = M4 * N;
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total; idx += stride) {
      const int64_t i = (idx % M4) * 4, j = idx / M4;
      const float4 x = *reinterpret_cast<const float4*>(src + i + j * lds);
      float4 h, l;
      h.x = rn_tf32(x.x); l.x = rn_tf32(x.x - h.x);
      h.y = rn_tf32(x.y); l.y = rn_tf32(x.y - h.y);
      h.z = rn_tf32(x.z); l.z = rn_tf32(x.z - h.z);
      h.w = rn_tf32(x.w); l.w = rn_tf32(x.w - h.w);
      *reinterpret_cast<float4*>(hi + i + j * ldh) = h;
      *reinterpret_cast<float4*>(lo + i + j * ldl) = l;
    }
    return;
  }
  for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < M * N; idx += stride) {
    const int64_t i = idx % M, j = idx / M;
    const float x = src[i + j * lds];
    const float h = rn_tf32(x);
    hi[i + j * ldh] = h;
    lo[i + j * ldl] = rn_tf32(x - h);
  }
}

cudaError_t launch_tf32_split(const float* src, int64_t lds, float* hi, int64_t ldh, float* lo, int64_t ldl,
                              int64_t M, int64_t N, int num_sms, cudaStream_t st) {
  if (M * N == 0) return cudaSuccess;
  const bool vec = M % 4 == 0 && lds % 4 == 0 && ldh % 4 == 0 && ldl % 4 == 0 &&
                   ((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(hi) |
                     reinterpret_cast<uintptr_t>(lo)) & 15) == 0;
  const int64_t work = vec ? (M / 4) * N : M * N;
  const int64_t blocks = std::min<int64_t>((work + 255) / 256, (int64_t)num_sms * 8);
  tf32_split_kernel<<<(unsigned)blocks, 256, 0, st>>>(src, lds, hi, ldh, lo, ldl, M, N, vec ? 1 : 0);
  return cudaGetLastError();
}

template <typename T>
__global__ void copy_cast_kernel(const float* __restrict__ src, int64_t lds, float* dst_f, int64_t ldf, T* dst_op,
                                 int64_t ldo, int64_t M, int64_t N) {
  const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= M * N) return;
  const int64_t i = idx % M, j = idx / M;
  const float v = src[i + j * lds];
  if (dst_f) dst_f[i + j * ldf] = v;
  if (dst_op) dst_op[i + j * ldo] = Elem<T>::store(v);
}

template <typename T>
cudaError_t launch_copy_cast(const float* src, int64_t lds, float* dst_f, int64_t ldf, T* dst_op, int64_t ldo,
                             int64_t M, int64_t N, cudaStream_t st) {
  const int64_t total = M * N;
  if (total == 0) return cudaSuccess;
  copy_cast_kernel<T><<<(unsigned)((total + 255) / 256), 256, 0, st>>>(src, lds, dst_f, ldf, dst_op, ldo, M, N);
  return cudaGetLastError();
}
template cudaError_t launch_copy_cast<__half>(const float*, int64_t, float*, int64_t, __half*, int64_t, int64_t,
                                              int64_t, cudaStream_t);
template cudaError_t launch_copy_cast<__nv_bfloat16>(const float*, int64_t, float*, int64_t, __nv_bfloat16*,
                                                     int64_t, int64_t, int64_t, cudaStream_t);
template cudaError_t launch_copy_cast<float>(const float*, int64_t, float*, int64_t, float*, int64_t, int64_t,
                                             int64_t, cudaStream_t);

// CGS2 leaf: R <- S R (both w x w upper triangular, column-major), one CTA, fixed-order sums.
__global__ void trmm_upper_kernel(const float* __restrict__ S, int64_t lds, float* R, int64_t ldr, int w) {
  __shared__ float sS[LEAF_MAX_W * LEAF_MAX_W], sR[LEAF_MAX_W * LEAF_MAX_W];
  for (int idx = threadIdx.x; idx < w * w; idx += blockDim.x) {
    const int i = idx % w, j = idx / w;
    sS[idx] = S[i + j * lds];
    sR[idx] = R[i + j * ldr];
  }
  __syncthreads();
  for (int idx = threadIdx.x; idx < w * w; idx += blockDim.x) {
    const int i = idx % w, j = idx / w;
    float acc = 0.0f;
    for (int k = i; k <= j; ++k) acc = fmaf(sS[i + k * w], sR[k + j * w], acc);
    R[i + j * ldr] = i <= j ? acc : 0.0f;
  }
}

cudaError_t launch_trmm_upper(const float* S, int64_t lds, float* R, int64_t ldr, int w, cudaStream_t st) {
  if (w < 1 || w > LEAF_MAX_W) return cudaErrorInvalidValue;
  trmm_upper_kernel<<<1, 512, 0, st>>>(S, lds, R, ldr, w);
  return cudaGetLastError();
}

template cudaError_t launch_gemm<__half>(bool, int, const CUtensorMap&, const CUtensorMap&, const GemmParams&, int,
                                   cudaStream_t, const CUtensorMap*, const CUtensorMap*, GemmExtra);
template cudaError_t launch_gemm<__nv_bfloat16>(bool, int, const CUtensorMap&, const CUtensorMap&, const GemmParams&, int,
                                   cudaStream_t, const CUtensorMap*, const CUtensorMap*, GemmExtra);
template cudaError_t launch_gemm<float>(bool, int, const CUtensorMap&, const CUtensorMap&, const GemmParams&, int,
                                   cudaStream_t, const CUtensorMap*, const CUtensorMap*, GemmExtra);
template cudaError_t launch_splitk_reduce<__half>(const float*, int64_t, int64_t, int, float*, int64_t,
                                                  int, __half*, int64_t, int64_t, int64_t, cudaStream_t);
template cudaError_t launch_splitk_reduce<__nv_bfloat16>(const float*, int64_t, int64_t, int, float*,
                                                         int64_t, int, __nv_bfloat16*, int64_t, int64_t,
                                                         int64_t, cudaStream_t);
template cudaError_t launch_splitk_reduce<float>(const float*, int64_t, int64_t, int, float*, int64_t,
                                                 int, float*, int64_t, int64_t, int64_t, cudaStream_t);

}  // namespace rgsqr
