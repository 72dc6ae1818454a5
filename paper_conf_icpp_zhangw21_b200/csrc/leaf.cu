// leaf.cu -- the leaf panel factorization: classical Gram-Schmidt, Eq. (1),
// CGS evaluation order (every r_ij = q_i^T a_j taken from the ORIGINAL column a_j,
// PAPER.md:109), for an m x w panel (w <= 64) held on chip.
//
// Mapping: a cooperative grid of G CTAs (one per SM); CTA g owns rows
// [g*RP, (g+1)*RP) of the panel, kept in shared memory as fp32 for the whole leaf.
// CGS needs reductions over all m rows; they are done in ROUNDS, one round per column:
//
//   round 0 : S = [ ||a_k||^2 (k < w),  a_0^T a_1 ]
//   round t : S = [ u_t^T u_t,  u_t^T a_{t+1},  q_{t-1}^T a_{t+1},  q_i^T a_{t+2} (i <= t-1) ]
//   after round t (every CTA, identical scalars):
//       r_tt = ||u_t||,  q_t = u_t / r_tt,  r_{t,t+1} = (u_t^T a_{t+1}) / r_tt,
//       u_{t+1} = w_{t+1} - q_{t-1} r_{t-1,t+1} - q_t r_{t,t+1},
//       w_{t+2} = a_{t+2} - sum_{i<=t-1} q_i r_{i,t+2}   (while round t+1 is in flight)
//
// i.e. the projection coefficient of the column just normalised is folded into the
// norm's reduction (q_t^T a = (u_t^T a) / r_tt), so each column costs ONE grid-wide
// reduction instead of two -- the same CGS quantities up to rounding order
// (reading R19).
//
// Exchange (rounds >= 1): every CTA red.add's each of its partials, converted to an exact
// fixed-point integer, into one 64-bit word per value that also counts arrivals; the
// value's thread in every CTA polls the word until all CTAs have added.  Integer sums are
// order-independent, so the result is deterministic.  Only the 4 values that depend on the
// previous round sit on the critical path; the others (q_i^T a_{t+2}, i <= t-2) are added
// two rounds early.  Round 0 uses a counter barrier + fixed-order gather of fp32 partials.
// Measured alternatives: scripts/barrier_bench.cu, scripts/exchange_bench.cu.
#include <type_traits>

#include "dtype.cuh"
#include "kernels.h"

namespace rgsqr {

static constexpr int LEAF_THREADS = 512;
static constexpr int LEAF_WARPS = LEAF_THREADS / 32;
static constexpr int GEMV_PARTS = LEAF_THREADS / 32;   // row parts of the local GEMV

__device__ __forceinline__ void st_relaxed_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.b64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ld_word(const unsigned long long* p, int sys) {
  if (!sys) return ld_relaxed_u64(p);
  unsigned long long v;
  asm volatile("ld.relaxed.sys.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

// Fixed-point exchange word: bits [53,64) count arrivals (<= 2047 = ranks x CTAs),
// bits [0,53) accumulate (v + 2^41) with |v| <= 2^41 per arrival (no carry into the count).
static constexpr int FX_CNT_SHIFT = 53;
static constexpr int FX_VBITS = 41;
static_assert((1 << (64 - FX_CNT_SHIFT)) - 1 == LEAF_MAX_ARRIVALS, "arrival count field width");
static_assert(LEAF_MAX_G <= LEAF_MAX_ARRIVALS, "one GPU's grid must fit the count field");

__device__ __forceinline__ void st_release_shared(int* p, int v) {
  asm volatile("st.release.cta.shared.b32 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(p)), "r"(v) : "memory");
}
__device__ __forceinline__ int ld_acquire_shared(const int* p) {
  int v;
  asm volatile("ld.acquire.cta.shared.b32 %0, [%1];" : "=r"(v) : "r"((unsigned)__cvta_generic_to_shared(p)) : "memory");
  return v;
}

// named barriers: the reducing warp waits for all threads, the others only arrive
__device__ __forceinline__ void bar_sync_n(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }
__device__ __forceinline__ void bar_arrive_n(int id, int n) { asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(n) : "memory"); }

__device__ __forceinline__ long long gtimer() {
  long long v;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(v));
  return v;
}

// exact power of two as a double (|e| < 1000)
__device__ __forceinline__ double pow2d(int e) { return __hiloint2double((1023 + e) << 20, 0); }

// per-phase cycle stamps of CTA p.dbg_cta (diagnostics; p.dbg == nullptr in production)
#define DBG_CTA p.dbg_cta
#define PRO_STAMP(i)                                                       \
  if (p.dbg != nullptr && blockIdx.x == DBG_CTA && threadIdx.x == 0) p.dbg[(size_t)LEAF_MAX_W * 16 + (i)] = clock64();
// bulk-group stamps (slots 8..13 of round t, thread 0 of the bulk group)
#define BULK_STAMP(i)                                                   \
  if (p.dbg != nullptr && blockIdx.x == DBG_CTA && btid == 0) p.dbg[(size_t)t * 16 + (i)] = clock64();
#define DBG_STAMP(i)                                           \
  if (p.dbg != nullptr && blockIdx.x == DBG_CTA && threadIdx.x == 0) \
    p.dbg[(size_t)t * 16 + (i)] = clock64();

// 16-byte vector load of consecutive storage elements widened to fp32.
template <typename T>
struct Vec;
template <>
struct Vec<__half> {
  static constexpr int N = 8;
  __device__ static void load(const __half* p, float* o) {
    const uint4 u = *reinterpret_cast<const uint4*>(p);
    const __half2* h = reinterpret_cast<const __half2*>(&u);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const float2 f = __half22float2(h[i]);
      o[2 * i] = f.x;
      o[2 * i + 1] = f.y;
    }
  }
};
template <>
struct Vec<__nv_bfloat16> {
  static constexpr int N = 8;
  __device__ static void load(const __nv_bfloat16* p, float* o) {
    const uint4 u = *reinterpret_cast<const uint4*>(p);
    const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const float2 f = __bfloat1622float2(h[i]);
      o[2 * i] = f.x;
      o[2 * i + 1] = f.y;
    }
  }
};
template <>
struct Vec<float> {
  static constexpr int N = 4;
  __device__ static void load(const float* p, float* o) {
    const float4 u = *reinterpret_cast<const float4*>(p);
    o[0] = u.x;
    o[1] = u.y;
    o[2] = u.z;
    o[3] = u.w;
  }
};

// store 4 consecutive rounded elements (8- or 16-byte aligned destination)
template <typename T>
__device__ __forceinline__ void store4(T* dst, float4 v);
template <>
__device__ __forceinline__ void store4<__half>(__half* dst, float4 v) {
  __half2 a = __floats2half2_rn(v.x, v.y), b = __floats2half2_rn(v.z, v.w);
  uint2 u;
  u.x = *reinterpret_cast<unsigned*>(&a);
  u.y = *reinterpret_cast<unsigned*>(&b);
  *reinterpret_cast<uint2*>(dst) = u;
}
template <>
__device__ __forceinline__ void store4<__nv_bfloat16>(__nv_bfloat16* dst, float4 v) {
  __nv_bfloat162 a = __floats2bfloat162_rn(v.x, v.y), b = __floats2bfloat162_rn(v.z, v.w);
  uint2 u;
  u.x = *reinterpret_cast<unsigned*>(&a);
  u.y = *reinterpret_cast<unsigned*>(&b);
  *reinterpret_cast<uint2*>(dst) = u;
}
template <>
__device__ __forceinline__ void store4<float>(float* dst, float4 v) {
  *reinterpret_cast<float4*>(dst) = v;
}

// CW: warps of the critical group (the other 16 - CW are the bulk group);
// NR: rows per critical-group thread (rows_per_cta <= 32 CW NR), their row state held in registers;
// NR == 0 ("tall" panels, rows_per_cta up to LEAF_MAX_RP_TALL): the critical group loops over any
// number of rows per thread with the row state read from the panel's shared-memory columns (u_t and
// q_t replace a_t in place), for panels whose slices exceed the register rows
template <typename T, int NR, int CW>
__global__ void __launch_bounds__(LEAF_THREADS, 1) leaf_cgs_kernel(LeafParams p) {
  extern __shared__ __align__(16) float sp[];      // [w][LD] column-major panel slice
  __shared__ float tot[2][LEAF_MAX_W + 2];         // reduced round vector, by parity of the round
  __shared__ float part[GEMV_PARTS][LEAF_MAX_W + 2];        // round 0 / lookahead partials
  __shared__ float part2[GEMV_PARTS / 2][LEAF_MAX_W];       // lookahead partials, second target
  __shared__ float cpart[GEMV_PARTS][8];                    // critical-dot partials
  __shared__ unsigned long long xprev[LEAF_XW_WORDS];      // last seen exchange words
  __shared__ __align__(16) float coef[3][LEAF_MAX_W + 4];   // r_{i,t+3}, i < t, by t mod 3
  __shared__ int exS[LEAF_MAX_W];                           // 2||a_j|| < 2^exS[j]
  __shared__ float tauc[LEAF_MAX_W];                        // breakdown thresholds
  __shared__ double fxs[LEAF_MAX_W][5], fxi[LEAF_MAX_W][5];  // fixed-point scales by (round, class)
  // the same scales in fp32 when 2^+-e is a normal float (else 0: the fp64 path is taken); scaling by a
  // power of two commutes with rounding, so both paths give bitwise-equal results for normal values
  __shared__ float fxsf[LEAF_MAX_W][5], fxif[LEAF_MAX_W][5];
  // last-seen exchange words persist across launches (words are never reset, see fx_exp)
  PRO_STAMP(0);
  if (p.dbg2 != nullptr && threadIdx.x == 0) {
    unsigned sm;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
    p.dbg2[(size_t)2 * LEAF_MAX_W * LEAF_MAX_G + blockIdx.x] = sm;
  }
  for (int i = threadIdx.x; i < LEAF_XW_WORDS; i += blockDim.x) xprev[i] = p.xprev_g[i];

  const int G = gridDim.x;
  const int g = blockIdx.x;
  const int w = p.w;
  const int RP = p.rows_per_cta;                   // rows owned by this CTA (max), multiple of 8
  const int LD = leaf_ld(RP);                      // smem column stride, == 4 (mod 32)
  const int64_t r0 = (int64_t)g * RP;
  const int64_t rem = p.m - r0;
  const int rows = rem <= 0 ? 0 : (rem < RP ? (int)rem : RP);
  const int rows4 = (rows + 3) & ~3;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  T* P = reinterpret_cast<T*>(p.P);

  // ---- load the slice: 16-byte vector loads (rows are 16-byte aligned), fp32 in smem ----
  {
    constexpr int V = Vec<T>::N;
    const int nvec = p.vec_ok ? rows / V : 0;
    // batches of B independent 16-byte loads per thread in flight before the converting stores
    constexpr int B = 8;
    for (int base = threadIdx.x; base < w * nvec; base += B * LEAF_THREADS) {
      uint4 raw[B];
#pragma unroll
      for (int u = 0; u < B; ++u) {
        const int idx = base + u * LEAF_THREADS;
        if (idx < w * nvec) {
          const int j = idx / nvec, i = (idx - j * nvec) * V;
          raw[u] = *reinterpret_cast<const uint4*>(P + r0 + i + (int64_t)j * p.ldp);
        }
      }
#pragma unroll
      for (int u = 0; u < B; ++u) {
        const int idx = base + u * LEAF_THREADS;
        if (idx < w * nvec) {
          const int j = idx / nvec, i = (idx - j * nvec) * V;
          float f[V];
          Vec<T>::load(reinterpret_cast<const T*>(&raw[u]), f);
#pragma unroll
          for (int e = 0; e < V; e += 4)
            *reinterpret_cast<float4*>(sp + j * LD + i + e) = make_float4(f[e], f[e + 1], f[e + 2], f[e + 3]);
        }
      }
    }
    const int span = LD - nvec * V;
    for (int idx = threadIdx.x; idx < w * span; idx += LEAF_THREADS) {
      const int j = idx / span, i = nvec * V + (idx - j * span);
      sp[j * LD + i] = i < rows ? Elem<T>::load(P[r0 + i + (int64_t)j * p.ldp]) : 0.0f;
    }
  }
  __syncthreads();
  PRO_STAMP(1);

  const float u_work = 5.9604645e-08f;             // 2^-24, fp32 accumulation
  // Bulk GEMV mapping: thread (kq = lane, part = warp) handles values kq and kq + 32
  // over row part `warp`.  8 consecutive kq read 8 different columns at the same row:
  // with LD == 4 (mod 32) the float4 reads are conflict-free; a shared y is broadcast.
  const int kq = lane;
  const int nv4 = rows4 / 4;
  const int per = (nv4 + GEMV_PARTS - 1) / GEMV_PARTS;
  const int v_lo = min(nv4, warp * per), v_hi = min(nv4, v_lo + per);

  // dot(x-col, y-col) over this thread's float4 rows
  auto dot4 = [&](int cx, int cy) {
    const float4* x = reinterpret_cast<const float4*>(sp + cx * LD);
    const float4* y = reinterpret_cast<const float4*>(sp + cy * LD);
    float s0 = 0.f, s1 = 0.f;
    for (int i = v_lo; i < v_hi; ++i) {
      const float4 a = x[i], b = y[i];
      s0 = fmaf(a.x, b.x, s0);
      s1 = fmaf(a.y, b.y, s1);
      s0 = fmaf(a.z, b.z, s0);
      s1 = fmaf(a.w, b.w, s1);
    }
    return s0 + s1;
  };
  // Fixed-point exchange (rounds t >= 1): value k of round t is scaled by 2^e with e chosen
  // from a bound on |partial| (column norms of round 0), rounded to an integer |v| <= 2^41
  // and added with ONE red.add.u64 per CTA to its word as
  //     (1 << 53) + (v + 2^41)          -- bits [53,64) count arrivals, low 53 bits sum
  // Integer addition is associative, so the total is independent of arrival order
  // (deterministic) and exact in fixed point; words are never reset: readers take the
  // difference with the value they saw at the previous use of the word.
  auto fx_exp = [&](int t, int k) -> int {
    // |partial| <= bound: ||a_t||^2, ||a_t|| ||a_{t+1}||, ||a_{t+1}||, ||a_{t+2}||, ||a_{t+3}|| for
    // value classes 0, 1, 2, 3, 4+ (u_t shrinks a_t, ||q_i|| <= 1); 2||a_j|| < 2^exS[j]
    if (k == 0) return FX_VBITS - 2 * exS[t];
    if (k == 1) return FX_VBITS - (exS[t] + exS[t + 1]);
    if (k == 2) return FX_VBITS - (exS[t + 1] + 1);
    if (k == 3) return FX_VBITS - (exS[t + 2] + 1);
    return FX_VBITS - (exS[t + 3] + 1);
  };
  // Words of round t: set t mod LEAF_XW_SETS (a round's words are reused only after every
  // CTA has read them: the lookahead values of round t are added two rounds early), one
  // 256-byte line per word so that concurrent atomics and polls land in different L2 slices.
  auto xw_index = [&](int t, int k) -> int { return (t & (LEAF_XW_SETS - 1)) * (LEAF_MAX_W + 2) + k; };
  // value -> fixed point (s * 2^e rounded to an integer) and back (total * 2^-e rounded to fp32)
  auto to_fx = [&](float s, float sf, double sd) -> long long {
    return sf != 0.0f ? __float2ll_rn(s * sf) : __double2ll_rn((double)s * sd);
  };
  auto from_fx = [&](long long total, float xf, double xd) -> float {
    if (xf != 0.0f) {
      const float v = __ll2float_rn(total) * xf;
      if (!(fabsf(v) < 1.17549435e-38f) || total == 0) return v;   // (subnormal results: the fp64 path)
    }
    return (float)((double)total * xd);
  };
  auto fx_add_scaled = [&](int t, int k, float s, float sf, double sd) {
    long long v = to_fx(s, sf, sd);
    const long long vb = 1ll << FX_VBITS;
    v = v > vb ? vb : (v < -vb ? -vb : v);
    const unsigned long long add = (1ull << FX_CNT_SHIFT) + (unsigned long long)(v + vb);
    const size_t off = (size_t)xw_index(t, k) * LEAF_XW_STRIDE;
    if (!p.sys) {
      asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p.xw + off), "l"(add) : "memory");
    } else {
      // row-sharded run: the same word on every GPU receives every CTA's partial
      for (int j = 0; j < p.nranks; ++j)
        asm volatile("red.relaxed.sys.global.add.u64 [%0], %1;" ::"l"(p.xw_peers[j] + off), "l"(add)
                     : "memory");
    }
  };
  auto fx_add = [&](int t, int k, float s) {
    const int c = k < 4 ? k : 4;
    fx_add_scaled(t, k, s, fxsf[t][c], fxs[t][c]);
  };
  // CTA total of values [0, n) of a [GEMV_PARTS][ld] partial buffer: 4 threads per value, each
  // adds a quarter of the parts, then a 2-level xor tree (fixed order).  Called by all threads;
  // the returned sum is valid on the thread with (threadIdx.x & 3) == 0 of value threadIdx.x >> 2.
  auto cta_sum = [&](const float* buf, int ld, int n) -> float {
    const int k = threadIdx.x >> 2, jq = threadIdx.x & 3;
    float s = 0.f;
    if (k < n) {
#pragma unroll
      for (int q = 0; q < GEMV_PARTS / 4; ++q) s += buf[(jq * (GEMV_PARTS / 4) + q) * ld + k];
    }
    s += __shfl_xor_sync(0xffffffffu, s, 1);
    s += __shfl_xor_sync(0xffffffffu, s, 2);
    return s;
  };

  // Round layout (t >= 1), R19/R22:
  //   [0] u_t.u_t   [1] u_t.a_{t+1}   [2] q_{t-1}.a_{t+1}   [3] q_{t-1}.a_{t+2}
  //   [4+i] q_i.a_{t+3}  (i <= t-1)
  // [0..3] and [4+(t-1)] are the CRITICAL values, formed in one pass over the rows right after
  // round t-1's scalars; [4+i], i <= t-2 ("lookahead") only need q's known two rounds earlier
  // and are computed AND added during round t-2's exchange.  After round t every CTA knows
  //   r_tt, r_{t,t+1} = [1]/r_tt, r_{t-1,t+1} = [2], r_{t-1,t+2} = [3], r_{i,t+3} = [4+i],
  // and forms  u_{t+1} = w_{t+1} - q_{t-2} r_{t-2,t+1} - q_{t-1} r_{t-1,t+1} - q_t r_{t,t+1},
  // where the projected column w_j = a_j - sum_{i <= j-4} q_i r_ij was formed two rounds
  // earlier (after round j-3) into a ring of LEAF_WRING smem columns, so that the projection
  // has a whole round of slack and never sits between an exchange and the next row pass.
  // The original a_j stay in place (CGS takes every r_ij from the original column,
  // PAPER.md:109) until u_j overwrites them.
  auto round_len = [&](int t) -> int {
    if (t == 0) return w + (w > 1 ? 1 : 0);
    if (t + 3 < w) return t + 4;
    if (t + 2 < w) return 4;
    if (t + 1 < w) return 3;
    return 1;
  };
  float* wring = sp + (size_t)w * LD;               // [LEAF_WRING][LD] projected columns
  // ---- round 0 vector: [ ||a_k||^2 (k < w), a_0^T a_1 ]: counter barrier + fixed-order gather
  //      (its column norms fix the fixed-point scales of the later rounds) ----
  // (r0_mode 2: the globally reduced round-0 vector is given in p.r0buf)
  if (p.r0_mode != 2) {
    const int L = round_len(0);
    if (p.r0_mode != 3) {   // (mode 3: the partials were written by the preceding fused node)
    for (int k = kq; k < L; k += 32) {
      int cx = k < w ? k : 0, cy = k < w ? k : 1;
      part[warp][k] = dot4(cx, cy);
    }
    __syncthreads();
    PRO_STAMP(8);
    const float s = cta_sum(&part[0][0], LEAF_MAX_W + 2, L);
    if ((threadIdx.x & 3) == 0 && (threadIdx.x >> 2) < L) p.partials[(size_t)(threadIdx.x >> 2) * G + g] = s;
    __syncthreads();
    PRO_STAMP(9);
    if (threadIdx.x == 0) {  // release: orders this CTA's partial stores (bar.sync cumulativity)
      asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(p.counter) : "memory");
      unsigned cv;
      do {
        asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(cv) : "l"(p.counter) : "memory");
      } while ((int)(cv - p.counter_target) < 0);   // (wrap-safe: the counter is never reset)
    }
    __syncthreads();
    PRO_STAMP(10);
    }
    constexpr int KPW = (LEAF_MAX_W + 2 + LEAF_WARPS - 1) / LEAF_WARPS;
    constexpr int QMAX = (LEAF_MAX_G + 31) / 32;
    float v[KPW][QMAX];
#pragma unroll
    for (int a = 0; a < KPW; ++a)
#pragma unroll
      for (int q = 0; q < QMAX; ++q) {
        const int k = warp + a * LEAF_WARPS, c = lane + 32 * q;
        v[a][q] = (k < L && c < G) ? __ldcg(p.partials + (size_t)k * G + c) : 0.0f;
      }
#pragma unroll
    for (int a = 0; a < KPW; ++a) {
      const int k = warp + a * LEAF_WARPS;
      if (k >= L) break;                               // warp-uniform
      float s2 = v[a][0];
#pragma unroll
      for (int q = 1; q < QMAX; ++q) s2 += v[a][q];
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) s2 += __shfl_xor_sync(0xffffffffu, s2, o);
      if (lane == 0) tot[0][k] = s2;
    }
    if (p.r0_mode == 1) {
      // round-0-only launch of a row-sharded run: hand the local vector to the host
      // (which all-reduces it across GPUs) and stop
      __syncthreads();
      if (g == 0 && threadIdx.x < L) p.r0buf[threadIdx.x] = tot[0][threadIdx.x];
      return;
    }
  } else if (threadIdx.x < round_len(0)) {
    tot[0][threadIdx.x] = p.r0buf[threadIdx.x];
  }
  __syncthreads();
  if (threadIdx.x < w) {
    const int k = threadIdx.x;
    const float s = tot[0][k];
    int ex;
    frexpf(2.0f * sqrtf(s), &ex);
    exS[k] = ex;
    tauc[k] = (float)p.m_global * u_work * sqrtf(s);
  }
  __syncthreads();
  PRO_STAMP(2);
  // fixed-point scales 2^fx_exp(t, class) and their inverses, value classes 0..4 (fx_exp)
  for (int i = threadIdx.x; i < w * 5; i += LEAF_THREADS) {
    const int t = i / 5, c = i - t * 5;
    const int need = c <= 1 ? t + c : (c == 2 ? t + 1 : (c == 3 ? t + 2 : t + 3));   // last column used
    const int e = need < w ? fx_exp(t, c) : 0;
    fxs[t][c] = pow2d(e);
    fxi[t][c] = pow2d(-e);
    fxsf[t][c] = (e > -120 && e < 120) ? __int_as_float((127 + e) << 23) : 0.0f;
    fxif[t][c] = (e > -120 && e < 120) ? __int_as_float((127 - e) << 23) : 0.0f;
  }
  // (the __syncthreads at the top of the round loop publishes exS / tauc)

  // Warp specialisation (the 3-deep round layout above makes it legal):
  //   CRITICAL group, warps [0, 8):  poll round t -> scalars -> row pass (u_{t+1}, q_t, round
  //     t+1's critical dots) -> publish -> poll round t+1 ...   (rows ctid + 256k)
  //   BULK group, warps [8, 16):  after q_t is in shared memory: round t+2's lookahead dots and
  //     the projection w_{t+3}, concurrently with the critical group's next rounds.
  // The groups hand off through producer/consumer named barriers (one per direction and
  // round parity, so that a group can never arrive twice on a barrier its partner has not
  // yet waited on -- each direction's round t+2 depends on the other direction's round t):
  //   BAR_Q + (t&1): critical arrives once q_0..q_t (and coef of round t) are in smem, the
  //                  bulk waits before its round t;
  //   BAR_W + (t&1): the bulk arrives after its round t (w_{t+3} in the ring), the critical
  //                  group waits before its row pass after round t+2.
  // Barriers order shared memory without draining the threads' outstanding global stores
  // (a release store would).  Within a group: named barrier 1 (critical), 3 (lookahead
  // reduction); CRIT_W reduces the critical partials, LA_W the lookahead partials.
  constexpr int GROUP = 32 * CW, GROUP_W = CW;                       // critical group
  constexpr int BULK = LEAF_THREADS - GROUP, BULK_W = LEAF_WARPS - CW;   // bulk group
  constexpr int CRIT_W = GROUP_W - 1, LA_W = LEAF_WARPS - 1;
  static_assert(BULK_W <= GEMV_PARTS / 2, "part2 holds one row per bulk warp");
  const bool is_crit = threadIdx.x < GROUP;
  const int crit_warps = rows >= GROUP ? GROUP_W : (rows + 31) / 32;   // critical warps owning rows
  PRO_STAMP(3);
  constexpr int BAR_Q = 4, BAR_W = 6;
  if (is_crit) {
    // row state of this thread's rows rr[j] = tid + 32 CW j, j < NR (NR == 0: none, see above)
    constexpr int NRA = NR > 0 ? NR : 1;
    int rr[NRA];
    bool vr[NRA];
    float ru[NRA], rq1[NRA], rq2[NRA], rq3[NRA], ra2[NRA], ra3[NRA];
#pragma unroll
    for (int j = 0; j < NR; ++j) {
      rr[j] = threadIdx.x + GROUP * j;
      vr[j] = rr[j] < rows;
      ru[j] = vr[j] ? sp[rr[j]] : 0.0f;                              // u_0 = a_0
      ra2[j] = (vr[j] && w > 2) ? sp[2 * LD + rr[j]] : 0.0f;
      ra3[j] = (vr[j] && w > 3) ? sp[3 * LD + rr[j]] : 0.0f;
      rq1[j] = rq2[j] = rq3[j] = 0.0f;
    }
    for (int t = 0; t < w; ++t) {
      DBG_STAMP(0);
      const float tau = tauc[t];   // (constant during the rounds: loaded before the exchange wait)
      if (t > 0) {
        // ---- round t's exchange: each of the (at most 4) values the scalars need is polled
        //      by its thread until all ranks x G CTAs have added; values [4+i] (coefficients
        //      of the projection) are polled by the bulk group ----
        // thread 4: r_{t-3,t+1} = value [4+(t-3)] of round t-2 (added by the bulk groups after
        // round t-3, so normally complete long before)
        const int L = min(round_len(t), 4);
        const bool late = threadIdx.x == 4 && t >= 3 && t + 1 < w;
        if (threadIdx.x < L || late) {
          const int k = late ? 4 + (t - 3) : threadIdx.x;
          const int tr = late ? t - 2 : t;
          const int widx = xw_index(tr, k);
          const unsigned cnt = (unsigned)(p.nranks * G);
          const unsigned long long* wp = p.xw + (size_t)widx * LEAF_XW_STRIDE;
          const unsigned long long prev = xprev[widx];
          unsigned long long now = ld_word(wp, p.sys), d = now - prev;
          long long spins = 0;
          while ((unsigned)(d >> FX_CNT_SHIFT) != cnt) {
            if (p.poll_sleep_ns) __nanosleep(p.poll_sleep_ns);
            now = ld_word(wp, p.sys);
            d = now - prev;
            if (++spins > (1ll << 22)) {            // ~seconds: a peer is missing -- fail, never hang
              atomicExch(p.breakdown, -2);
              break;
            }
          }
          xprev[widx] = now;
          if (p.dbg2 != nullptr && k == 0) p.dbg2[((size_t)g * LEAF_MAX_W + t) * 2 + 1] = gtimer();
          const long long total = (long long)(d & ((1ull << FX_CNT_SHIFT) - 1)) - (long long)cnt * (1ll << FX_VBITS);
          const float val = from_fx(total, fxif[tr][k < 4 ? k : 4], fxi[tr][k < 4 ? k : 4]);
          tot[t & 1][late ? 4 : k] = val;
        }
      }
      // the row pass after round t reads w_{t+1}, projected by the bulk after round t-2: wait
      // for that bulk round (this barrier also publishes the polled values to the group)
      if (t >= 2 && t + 1 < w)
        bar_sync_n(BAR_W + (t & 1), LEAF_THREADS);
      else
        bar_sync_n(1, GROUP);
      DBG_STAMP(1);
      // ---- scalars (every thread, identical): r_tt, 1/r_tt, r_{t,t+1}, r_{t-1,t+1}, r_{t-2,t+1} ----
      const bool more = t + 1 < w;
      const float* tt = tot[t & 1];
      const float uu = tt[0];
      const float ua = (t == 0) ? ((w > 1) ? tt[w] : 0.0f) : (more ? tt[1] : 0.0f);
      const float c1 = (t >= 1 && more) ? tt[2] : 0.0f;    // r_{t-1,t+1} = q_{t-1}^T a_{t+1}
      const float c2 = (t >= 2 && more) ? tot[(t - 1) & 1][3] : 0.0f;   // r_{t-2,t+1} (round t-1)
      const float c3 = (t >= 3 && more) ? tt[4] : 0.0f;    // r_{t-3,t+1} (round t-2)
      float rtt = sqrtf(uu);
      const bool bad = !(rtt > tau) || !isfinite(rtt);
      const float inv = bad ? 0.0f : __frcp_rn(rtt);     // == 1/rtt (correctly rounded)
      if (bad) rtt = 0.0f;
      const float ct = ua * inv;                            // r_{t,t+1}
      // this round's R entries (CTA 0), written after the CTA has published round t+1's values:
      // stores on CTA 0's critical path made it the last publisher of every round
      auto write_r = [&]() {
        if (g != 0) return;
        if (threadIdx.x == 0) {
          p.R[t + (int64_t)t * p.ldr] = rtt;
          if (bad) atomicMin(p.breakdown, (int)(p.col_offset + t));
          if (more) p.R[t + (int64_t)(t + 1) * p.ldr] = ct;
        } else if (threadIdx.x == 1) {
          if (t >= 1 && more) p.R[(t - 1) + (int64_t)(t + 1) * p.ldr] = c1;
          if (t >= 1 && t + 2 < w) p.R[(t - 1) + (int64_t)(t + 2) * p.ldr] = tt[3];   // r_{t-1,t+2}
          if (t >= 3 && more) p.R[(t - 3) + (int64_t)(t + 1) * p.ldr] = c3;
        }
        if (threadIdx.x > t && threadIdx.x < w) p.R[threadIdx.x + (int64_t)t * p.ldr] = 0.0f;
      };
      DBG_STAMP(2);
      // ---- one pass over this thread's (at most 2) rows, both rows interleaved, the row
      //      state in registers (u_t, q_{t-1}, q_{t-2}, a_{t+2}, a_{t+3}):
      //      q_t = u_t / r_tt (to smem for the bulk group, rounded to global Q),
      //      u_{t+1} = w_{t+1} - q_{t-2} r_{t-2,t+1} - q_{t-1} r_{t-1,t+1} - q_t r_{t,t+1}
      //      (w_{t+1} = a_{t+1} for t+1 <= 3), and round t+1's critical dots
      //      u_{t+1}.u_{t+1}, u_{t+1}.a_{t+2}, q_t.a_{t+2}, q_t.a_{t+3}, q_t.a_{t+4} ----
      const bool h2 = t + 2 < w, h3 = t + 3 < w, h4 = t + 4 < w;
      float s0, s1, s2, s3, s4;
      if constexpr (NR == 0) {
        // tall panel: rows tid + 32 CW j of the shared-memory slice, same arithmetic as below;
        // u_{t+1} replaces a_{t+1} in column t+1 (no reader of a_{t+1} is left: the critical dots
        // use a_{t+2..t+4}, the bulk round t-1 still running reads a_{t+2..t+4} and q's)
        const float* wsrc = (t + 1 <= 4) ? sp + (more ? t + 1 : t) * LD : wring + ((t + 1) % LEAF_WRING) * LD;
        float* ut = sp + t * LD;
        const float* q1p = sp + (t >= 1 ? t - 1 : t) * LD;
        const float* q2p = sp + (t >= 2 ? t - 2 : t) * LD;
        const float* q3p = sp + (t >= 3 ? t - 3 : t) * LD;
        const float* a2p = sp + (h2 ? t + 2 : t) * LD;
        const float* a3p = sp + (h3 ? t + 3 : t) * LD;
        const float* a4p = sp + (h4 ? t + 4 : t) * LD;
        float* un = sp + (more ? t + 1 : t) * LD;
        s0 = s1 = s2 = s3 = s4 = 0.0f;
#pragma unroll 2
        for (int r = threadIdx.x; r < rows; r += GROUP) {
          const float u = ut[r];
          const float q1 = t >= 1 ? q1p[r] : 0.0f, q2 = t >= 2 ? q2p[r] : 0.0f, q3 = t >= 3 ? q3p[r] : 0.0f;
          const float wv = more ? wsrc[r] : 0.0f;
          const float a2 = h2 ? a2p[r] : 0.0f, a3 = h3 ? a3p[r] : 0.0f, a4 = h4 ? a4p[r] : 0.0f;
          const float q = u * inv;
          float x = fmaf(-q3, c3, wv);
          x = fmaf(-q2, c2, x);
          x = fmaf(-q1, c1, x);
          const float av = fmaf(-q, ct, x);
          ut[r] = q;
          if (more) un[r] = av;
          s0 = fmaf(av, av, s0);
          s1 = fmaf(av, a2, s1);
          s2 = fmaf(q, a2, s2);
          s3 = fmaf(q, a3, s3);
          s4 = fmaf(q, a4, s4);
        }
      } else {
        const float* wsrc = (t + 1 <= 4) ? sp + (more ? t + 1 : t) * LD : wring + ((t + 1) % LEAF_WRING) * LD;
        const float* a4p = sp + (h4 ? t + 4 : t) * LD;
        float* ut = sp + t * LD;
        float wv[NR], a4v[NR], q[NR], av[NR];
#pragma unroll
        for (int j = 0; j < NR; ++j) {
          const int r = rr[j];
          wv[j] = (vr[j] && more) ? wsrc[r] : 0.0f;
          a4v[j] = (vr[j] && h4) ? a4p[r] : 0.0f;
        }
#pragma unroll
        for (int j = 0; j < NR; ++j) {
          q[j] = ru[j] * inv;
          float x = fmaf(-rq3[j], c3, wv[j]);
          x = fmaf(-rq2[j], c2, x);
          x = fmaf(-rq1[j], c1, x);
          av[j] = fmaf(-q[j], ct, x);
        }
#pragma unroll
        for (int j = 0; j < NR; ++j)
          if (vr[j]) ut[rr[j]] = q[j];   // (global Q: stored from registers in the exchange wait)
        s0 = s1 = s2 = s3 = s4 = 0.0f;
#pragma unroll
        for (int j = 0; j < NR; ++j) {
          s0 = fmaf(av[j], av[j], s0);
          s1 = fmaf(av[j], ra2[j], s1);
          s2 = fmaf(q[j], ra2[j], s2);
          s3 = fmaf(q[j], ra3[j], s3);
          s4 = fmaf(q[j], a4v[j], s4);   // q_t.a_{t+4}: round t+1's [4+t], reduced after publishing
        }
#pragma unroll
        for (int j = 0; j < NR; ++j) {
          rq3[j] = rq2[j];
          rq2[j] = rq1[j];
          rq1[j] = q[j];
          ru[j] = av[j];
          ra2[j] = ra3[j];
          ra3[j] = a4v[j];
        }
      }
      if (!more) {
        write_r();
        // the last column: its rows of Q straight from registers (tall: from this thread's smem rows)
        if constexpr (NR == 0) {
          for (int r = threadIdx.x; r < rows; r += GROUP) P[r0 + r + (int64_t)t * p.ldp] = Elem<T>::store(sp[t * LD + r]);
        }
#pragma unroll
        for (int j = 0; j < NR; ++j)
          if (vr[j]) P[r0 + rr[j] + (int64_t)t * p.ldp] = Elem<T>::store(rq1[j]);
        break;
      }
      // the critical reducer's lane 4c (c < 5) adds value c of round t+1: its fixed-point scale now
      const int n_crit = !h2 ? 1 : (!h3 ? 3 : 4);   // critical values of round t+1
      double crit_scale = 0.0;
      float crit_scale_f = 0.0f;
      if (warp == CRIT_W && (lane & 7) == 0 && (lane >> 3) < n_crit) {
        crit_scale = fxs[t + 1][lane >> 3];
        crit_scale_f = fxsf[t + 1][lane >> 3];
      }
      // warp sums of the 5 critical values: a transposing butterfly (6 shuffles) leaves value k
      // < 4 in lane 8k, an xor tree the fifth (fixed tree per value)
      {
        const bool b16 = lane & 16, b8 = lane & 8;
        float k0 = b16 ? s2 : s0, k1 = b16 ? s3 : s1;
        const float x0 = b16 ? s0 : s2, x1 = b16 ? s1 : s3;
        k0 += __shfl_xor_sync(0xffffffffu, x0, 16);
        k1 += __shfl_xor_sync(0xffffffffu, x1, 16);
        float kk = b8 ? k1 : k0;
        kk += __shfl_xor_sync(0xffffffffu, b8 ? k0 : k1, 8);
        kk += __shfl_xor_sync(0xffffffffu, kk, 4);
        kk += __shfl_xor_sync(0xffffffffu, kk, 2);
        kk += __shfl_xor_sync(0xffffffffu, kk, 1);
        if ((lane & 7) == 0) cpart[warp][lane >> 3] = kk;
      }
      DBG_STAMP(3);
      bar_sync_n(1, GROUP);
      // q_0..q_t (and coef of round t) are in smem: release the bulk group for round t
      if (t + 3 < w) bar_arrive_n(BAR_Q + (t & 1), LEAF_THREADS);
      // ---- publish round t+1's critical values [0..3] and [4 + t] (warp CRIT_W) ----
      if (warp == CRIT_W) {
        const int c = lane >> 3, j = lane & 7;
        float s = j < crit_warps ? cpart[j][c] : 0.0f;
        s += __shfl_xor_sync(0xffffffffu, s, 4);
        s += __shfl_xor_sync(0xffffffffu, s, 2);
        s += __shfl_xor_sync(0xffffffffu, s, 1);
        if (j == 0 && c < n_crit) fx_add_scaled(t + 1, c, s, crit_scale_f, crit_scale);
        if (p.dbg != nullptr && blockIdx.x == DBG_CTA && lane == 0) p.dbg[(size_t)t * 16 + 7] = clock64();
        if (p.dbg2 != nullptr && lane == 0) p.dbg2[((size_t)g * LEAF_MAX_W + t) * 2 + 0] = gtimer();
      }
      DBG_STAMP(4);
      write_r();
      // ---- inside round t+1's exchange wait: q_t.a_{t+4} (round t+1's value [4+t], read by this
      //      group after round t+3) reduced and added off the critical chain ----
      if (h4) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) s4 += __shfl_xor_sync(0xffffffffu, s4, o);
        if (lane == 0) cpart[warp][4] = s4;
        bar_sync_n(1, GROUP);
        if (warp == CRIT_W && lane == 0) {
          float v = 0.f;
          for (int j = 0; j < crit_warps; ++j) v += cpart[j][4];
          fx_add(t + 1, 4 + t, v);
        }
      }
      // q_t of this thread's rows to global memory (rounded once), inside the exchange wait
      if constexpr (NR == 0) {
        for (int r = threadIdx.x; r < rows; r += GROUP) P[r0 + r + (int64_t)t * p.ldp] = Elem<T>::store(sp[t * LD + r]);
      }
#pragma unroll
      for (int j = 0; j < NR; ++j)
        if (vr[j]) P[r0 + rr[j] + (int64_t)t * p.ldp] = Elem<T>::store(rq1[j]);
    }
  } else {
    // ---- BULK group: for each round t, after q_t is in smem:
    //      (a) round t+2's lookahead values q_i.a_{t+5}, i <= t (index 4 + i), over this warp's
    //          32-row blocks (lane = i), reduced by warp LA_W and added to round t+2's words;
    //      (b) w_{t+3} = a_{t+3} - sum_{i <= t-1} q_i r_{i,t+3}  (coefficients of round t) into
    //          the ring; the critical group first reads it after round t+2 ----
    const int btid = threadIdx.x - GROUP, bw = warp - GROUP_W;
    // the last bulk warp owns no projection row pairs: it can reduce the lookahead partials
    // while the others project
    const bool la_free = (NR * GROUP + 2 * BULK - 1) / (2 * BULK) == 1 && (rows + 1) / 2 <= BULK - 32;
    for (int t = 0; t + 3 < w; ++t) {
      BULK_STAMP(13);
      bar_sync_n(BAR_Q + (t & 1), LEAF_THREADS);
      BULK_STAMP(8);
      // round t's values [4+i] = r_{i,t+3}, i <= t-1: round t is complete (the critical group
      // has seen it); the loads are issued now and checked after the dot products below
      const int pk = 4 + btid;
      const int pidx = xw_index(t, pk);
      const unsigned long long* pwp = p.xw + (size_t)pidx * LEAF_XW_STRIDE;
      unsigned long long pnow = 0;
      if (btid < t - 1) pnow = ld_word(pwp, p.sys);
      // (a) lookahead GEMV, every other round for two target columns (each q_i read once):
      //     even t: round t+1's [4+i] = q_i.a_{t+4}, i <= t-1, and round t+2's [4+i] =
      //     q_i.a_{t+5}, i <= t (lane = i).  Round t+1's [4+t] comes from the critical group.
      const bool ev = (t & 1) == 0;
      const bool g1 = ev && t >= 1 && t + 4 < w, g2 = ev && t + 5 < w;
      if (g1 || g2) {
        const int cnt1 = g1 ? t : 0, cnt2 = g2 ? t + 1 : 0;
        const int cnt = max(cnt1, cnt2);
        const bool ha = kq < cnt, hb = kq + 32 < cnt;
        float a0 = 0.f, a1 = 0.f, b0 = 0.f, b1 = 0.f, c0 = 0.f, c1 = 0.f, d0 = 0.f, d1 = 0.f;
        if (ha && !(p.skip & 2)) {
          const float4* y1 = reinterpret_cast<const float4*>(sp + (g1 ? t + 4 : t) * LD);
          const float4* y2 = reinterpret_cast<const float4*>(sp + (g2 ? t + 5 : t) * LD);
          const float4* xa = reinterpret_cast<const float4*>(sp + kq * LD);
          const float4* xb = reinterpret_cast<const float4*>(sp + (hb ? kq + 32 : kq) * LD);
          // 32-row blocks: the smem slice is zero-padded to a multiple of 32 rows (leaf_ld).  The second
          // column (lane + 32) is taken warp-uniformly when any lane has one (lanes without it compute
          // an ignored partial), so the unrolled loop has no branch and its loads can be hoisted
          auto gemv = [&](auto second) {
            for (int base = 8 * bw; base < nv4; base += 8 * BULK_W) {
#pragma unroll
              for (int i = base; i < base + 8; ++i) {
                const float4 u = y1[i], v = y2[i], a = xa[i];
                a0 = fmaf(a.x, u.x, a0);
                a1 = fmaf(a.y, u.y, a1);
                a0 = fmaf(a.z, u.z, a0);
                a1 = fmaf(a.w, u.w, a1);
                c0 = fmaf(a.x, v.x, c0);
                c1 = fmaf(a.y, v.y, c1);
                c0 = fmaf(a.z, v.z, c0);
                c1 = fmaf(a.w, v.w, c1);
                if constexpr (decltype(second)::value) {
                  const float4 bb = xb[i];
                  b0 = fmaf(bb.x, u.x, b0);
                  b1 = fmaf(bb.y, u.y, b1);
                  b0 = fmaf(bb.z, u.z, b0);
                  b1 = fmaf(bb.w, u.w, b1);
                  d0 = fmaf(bb.x, v.x, d0);
                  d1 = fmaf(bb.y, v.y, d1);
                  d0 = fmaf(bb.z, v.z, d0);
                  d1 = fmaf(bb.w, v.w, d1);
                }
              }
            }
          };
          if (cnt > 32)
            gemv(std::true_type{});
          else
            gemv(std::false_type{});
        }
        part[bw][kq] = a0 + a1;
        part[bw][kq + 32] = b0 + b1;
        part2[bw][kq] = c0 + c1;
        part2[bw][kq + 32] = d0 + d1;
      }
      BULK_STAMP(9);
      // reduction of the lookahead partials by warp LA_W (while the others project, when
      // LA_W owns no projection rows)
      auto la_reduce = [&]() {
        const int cnt1 = g1 ? t : 0, cnt2 = g2 ? t + 1 : 0;
        float sa = 0.f, sb = 0.f, sc = 0.f, sd = 0.f;
#pragma unroll
        for (int v = 0; v < BULK_W; ++v) {
          sa += part[v][lane];
          sb += part[v][lane + 32];
          sc += part2[v][lane];
          sd += part2[v][lane + 32];
        }
        if (lane < cnt1) fx_add(t + 1, 4 + lane, sa);
        if (lane + 32 < cnt1) fx_add(t + 1, 4 + lane + 32, sb);
        if (lane < cnt2) fx_add(t + 2, 4 + lane, sc);
        if (lane + 32 < cnt2) fx_add(t + 2, 4 + lane + 32, sd);
      };
      const bool la_work = g1 || g2;
      if (la_work) {
        if (warp == LA_W) {
          bar_sync_n(3, BULK);
          if (!la_free) la_reduce();
        } else {
          bar_arrive_n(3, BULK);
        }
      }
      if (btid < t - 1) {
        const unsigned cnt = (unsigned)(p.nranks * G);
        const unsigned long long prev = xprev[pidx];
        unsigned long long d = pnow - prev;
        long long spins = 0;
        while ((unsigned)(d >> FX_CNT_SHIFT) != cnt) {
          pnow = ld_word(pwp, p.sys);
          d = pnow - prev;
          if (++spins > (1ll << 22)) {
            atomicExch(p.breakdown, -2);
            break;
          }
        }
        xprev[pidx] = pnow;
        const long long total = (long long)(d & ((1ull << FX_CNT_SHIFT) - 1)) - (long long)cnt * (1ll << FX_VBITS);
        const float val = from_fx(total, fxif[t][4], fxi[t][4]);
        coef[t % 3][btid] = val;
        if (g == 0) p.R[btid + (int64_t)(t + 3) * p.ldr] = val;
      }
      if (!la_free) {
        bar_sync_n(2, BULK);
      } else if (warp != LA_W) {
        bar_sync_n(2, BULK - 32);
      } else if (la_work) {
        la_reduce();
      }
      BULK_STAMP(10);
      if (t >= 2 && !(p.skip & 4) && !(la_free && warp == LA_W)) {
        // thread-per-row: w_{t+3}[r] = a_{t+3}[r] - sum_{i < t} q_i[r] r_{i,t+3}  (two fixed-order
        // partial sums)
        const float* cf = coef[t % 3];
        const float* an = sp + (t + 3) * LD;
        float* wd = wring + ((t + 3) % LEAF_WRING) * LD;
        // row pairs (2 pi, 2 pi + 1), pi = btid + BULK (j + NP c): float2 loads, 4 independent chains;
        // tall panels take their row pairs in chunks c of NP per thread
        constexpr int NP = NR > 0 ? (NR * GROUP + 2 * BULK - 1) / (2 * BULK) : 4;
        const int npairs = (rows + 1) / 2;
        const int nchunk = NR > 0 ? 1 : (npairs + NP * BULK - 1) / (NP * BULK);
        for (int ch = 0; ch < nchunk; ++ch) {
        float2 e0[NP], e1[NP];
        int pb[NP];
#pragma unroll
        for (int j = 0; j < NP; ++j) {
          e0[j] = e1[j] = make_float2(0.f, 0.f);
          pb[j] = 2 * min(btid + BULK * (j + NP * ch), LD / 2 - 1);   // pairs >= npairs: computed, not stored
        }
        int k = 0;
#pragma unroll 2
        for (; k + 4 <= t - 1; k += 4) {
          const float4 c0 = *reinterpret_cast<const float4*>(cf + k);
#pragma unroll
          for (int j = 0; j < NP; ++j) {
            const float2 x0 = *reinterpret_cast<const float2*>(sp + (k + 0) * LD + pb[j]);
            const float2 x1 = *reinterpret_cast<const float2*>(sp + (k + 1) * LD + pb[j]);
            const float2 x2 = *reinterpret_cast<const float2*>(sp + (k + 2) * LD + pb[j]);
            const float2 x3 = *reinterpret_cast<const float2*>(sp + (k + 3) * LD + pb[j]);
            e0[j].x = fmaf(x0.x, c0.x, e0[j].x);
            e0[j].y = fmaf(x0.y, c0.x, e0[j].y);
            e1[j].x = fmaf(x1.x, c0.y, e1[j].x);
            e1[j].y = fmaf(x1.y, c0.y, e1[j].y);
            e0[j].x = fmaf(x2.x, c0.z, e0[j].x);
            e0[j].y = fmaf(x2.y, c0.z, e0[j].y);
            e1[j].x = fmaf(x3.x, c0.w, e1[j].x);
            e1[j].y = fmaf(x3.y, c0.w, e1[j].y);
          }
        }
        for (; k < t - 1; ++k) {
          const float c0 = cf[k];
#pragma unroll
          for (int j = 0; j < NP; ++j) {
            const float2 x0 = *reinterpret_cast<const float2*>(sp + k * LD + pb[j]);
            e0[j].x = fmaf(x0.x, c0, e0[j].x);
            e0[j].y = fmaf(x0.y, c0, e0[j].y);
          }
        }
#pragma unroll
        for (int j = 0; j < NP; ++j)
          if (btid + BULK * (j + NP * ch) < npairs) {
            const float2 av = *reinterpret_cast<const float2*>(an + pb[j]);
            *reinterpret_cast<float2*>(wd + pb[j]) = make_float2(av.x - (e0[j].x + e1[j].x), av.y - (e0[j].y + e1[j].y));
          }
        }
      }
      BULK_STAMP(11);
      bar_arrive_n(BAR_W + (t & 1), LEAF_THREADS);
      BULK_STAMP(12);
    }
  }
  PRO_STAMP(4);
  __syncthreads();
  PRO_STAMP(5);
  PRO_STAMP(6);
  // every CTA ends with the same last-seen words; CTA 0 persists them for the next launch
  if (g == 0)
    for (int i = threadIdx.x; i < LEAF_XW_WORDS; i += blockDim.x) p.xprev_g[i] = xprev[i];
}

template <typename T, int NR, int CW>
static cudaError_t launch_leaf_nr(const LeafParams& p, int grid, cudaStream_t st) {
  const size_t smem = (size_t)(p.w + LEAF_WRING) * leaf_ld(p.rows_per_cta) * sizeof(float);
  static size_t attr_smem = 0;
  if (smem > attr_smem) {
    cudaError_t e = cudaFuncSetAttribute(leaf_cgs_kernel<T, NR, CW>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)smem);
    if (e != cudaSuccess) return e;
    attr_smem = smem;
  }
  // round 0's counter barrier (modes 0 and 1) waits for G more arrivals than all earlier launches
  // enqueued on this counter: no per-launch reset (a memset node per leaf)
  LeafParams q = p;
  const bool barrier = q.r0_mode == 0 || q.r0_mode == 1;
  if (barrier) q.counter_target = *p.counter_host + (unsigned)grid;
  cudaError_t e;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(LEAF_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  e = cudaLaunchKernelEx(&cfg, leaf_cgs_kernel<T, NR, CW>, q);
  if (e == cudaSuccess && barrier) *p.counter_host += (unsigned)grid;   // (only launched arrivals count)
  return e;
}

template <typename T>
cudaError_t launch_leaf(const LeafParams& p, int grid, cudaStream_t st) {
  // 8 critical + 8 bulk warps (4 + 12 measured slower at 448 rows per CTA)
  if (p.rows_per_cta <= 512) return launch_leaf_nr<T, 2, 8>(p, grid, st);
  if (p.rows_per_cta <= 1024) return launch_leaf_nr<T, 4, 8>(p, grid, st);
  if (p.rows_per_cta <= 2048) return launch_leaf_nr<T, 8, 8>(p, grid, st);
  if (p.rows_per_cta <= LEAF_MAX_RP_TALL) return launch_leaf_nr<T, 0, 8>(p, grid, st);   // tall panel
  return cudaErrorInvalidValue;   // rows_per_cta > LEAF_MAX_RP_TALL: rejected by op_leaf
}

int leaf_max_smem_rows(int w) { return (int)((LEAF_SMEM_BUDGET) / ((size_t)(w + LEAF_WRING) * sizeof(float))); }

template cudaError_t launch_leaf<__half>(const LeafParams&, int, cudaStream_t);
template cudaError_t launch_leaf<__nv_bfloat16>(const LeafParams&, int, cudaStream_t);
template cudaError_t launch_leaf<float>(const LeafParams&, int, cudaStream_t);

}  // namespace rgsqr
