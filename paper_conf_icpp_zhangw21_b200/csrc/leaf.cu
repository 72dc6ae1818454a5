// leaf.cu -- the leaf panel factorization: classical Gram-Schmidt, Eq. (1),
// CGS evaluation order (every r_ij = q_i^T a_j taken from the ORIGINAL column a_j,
// PAPER.md:109), for an m x w panel (w <= 64) held on chip.
//
// Mapping: a cooperative grid of G CTAs (one per SM); CTA g owns rows
// [g*RP, (g+1)*RP) of the panel, kept in shared memory as fp32 for the whole leaf.
// CGS needs reductions over all m rows; they are done in ROUNDS, one round per column:
//
//   round 0 : S = [ ||a_k||^2 (k < w),  a_0^T a_1 ]
//   round t : S = [ u_t^T u_t,  u_t^T a_{t+1},  q_i^T a_{t+1} (i < t) ]
//   after round t (every CTA, identical scalars):
//       r_tt = ||u_t||,  q_t = u_t / r_tt,  r_{t,t+1} = (u_t^T a_{t+1}) / r_tt,
//       r_{i,t+1} = q_i^T a_{t+1} (i < t),  u_{t+1} = a_{t+1} - sum_{i<=t} q_i r_{i,t+1}.
//
// i.e. the projection coefficient of the column just normalised is folded into the
// norm's reduction (q_t^T a = (u_t^T a) / r_tt), so each column costs ONE grid-wide
// reduction instead of two -- the same CGS quantities up to rounding order
// (reading R19).
//
// Exchange per round: each CTA writes its partial vector (fp32) to global memory,
// arrives on a counter (release) and spins on it (acquire); then every CTA loads the
// G partials of each value (all loads of a warp issued together) and sums them in the
// same fixed order (deterministic, no float atomics).  Measured alternatives
// (scripts/barrier_bench.cu, RGSQR_LEAF_DEBUG stamps): per-word round tags avoid the
// counter but flood L2 with spinning loads (4x slower gather).
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

// exact power of two as a double (|e| < 1000)
__device__ __forceinline__ double pow2d(int e) { return __hiloint2double((1023 + e) << 20, 0); }

// per-phase cycle stamps of CTA p.dbg_cta (diagnostics; p.dbg == nullptr in production)
#define DBG_CTA p.dbg_cta
#define DBG_STAMP(i)                                           \
  if (p.dbg != nullptr && blockIdx.x == DBG_CTA && threadIdx.x == 0) \
    p.dbg[(size_t)t * 8 + (i)] = clock64();

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

// column pair (x, y) whose dot product is value k of round t
__device__ __forceinline__ void round_operands(int t, int w, int k, int& cx, int& cy) {
  if (t == 0) {
    if (k < w) { cx = k; cy = k; }                     // ||a_k||^2
    else { cx = 0; cy = 1; }                           // a_0^T a_1
  } else {
    if (k == 0) { cx = t; cy = t; }                    // u_t^T u_t
    else if (k == 1) { cx = t; cy = t + 1; }           // u_t^T a_{t+1}
    else { cx = k - 2; cy = t + 1; }                   // q_i^T a_{t+1}
  }
}

template <typename T>
__global__ void __launch_bounds__(LEAF_THREADS, 1) leaf_cgs_kernel(LeafParams p) {
  extern __shared__ __align__(16) float sp[];      // [w][LD] column-major panel slice
  __shared__ float tot[LEAF_MAX_W + 2];            // reduced round vector
  __shared__ float anorm2[LEAF_MAX_W];             // ||a_k||^2 (breakdown threshold)
  __shared__ float part[2][GEMV_PARTS][LEAF_MAX_W + 2];     // by round parity
  __shared__ unsigned long long xprev[LEAF_XW_WORDS];      // last seen exchange words
  __shared__ __align__(16) float coef[2][LEAF_MAX_W + 4];   // r_{i,t+2}, i < t, by parity of t
  __shared__ int exS[LEAF_MAX_W];                           // 2||a_j|| < 2^exS[j]
  __shared__ float tauc[LEAF_MAX_W];                        // breakdown thresholds
  // last-seen exchange words persist across launches (words are never reset, see fx_exp)
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
    for (int idx = threadIdx.x; idx < w * nvec; idx += LEAF_THREADS) {
      const int j = idx / nvec, i = (idx - j * nvec) * V;
      float f[V];
      Vec<T>::load(P + r0 + i + (int64_t)j * p.ldp, f);
#pragma unroll
      for (int e = 0; e < V; e += 4)
        *reinterpret_cast<float4*>(sp + j * LD + i + e) = make_float4(f[e], f[e + 1], f[e + 2], f[e + 3]);
    }
    const int span = LD - nvec * V;
    for (int idx = threadIdx.x; idx < w * span; idx += LEAF_THREADS) {
      const int j = idx / span, i = nvec * V + (idx - j * span);
      sp[j * LD + i] = i < rows ? Elem<T>::load(P[r0 + i + (int64_t)j * p.ldp]) : 0.0f;
    }
  }
  __syncthreads();

  const float u_work = 5.9604645e-08f;             // 2^-24, fp32 accumulation
  // Bulk GEMV mapping: thread (kq = lane, part = warp) handles values kq and kq + 32
  // over row part `warp`.  8 consecutive kq read 8 different columns at the same row:
  // with LD == 4 (mod 32) the float4 reads are conflict-free; a shared y is broadcast.
  const int kq = lane;
  const int nv4 = rows4 / 4;
  const int per = (nv4 + GEMV_PARTS - 1) / GEMV_PARTS;
  const int v_lo = min(nv4, warp * per), v_hi = min(nv4, v_lo + per);
  // critical-dot mapping: warp = row part, lanes stride the part's rows
  const int c_lo = v_lo * 4, c_hi = min(rows, v_hi * 4);

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
  // warp-cooperative dots over the warp's row part (lanes stride rows, xor-trees):
  // u^T u, u^T a, q^T a in one pass (u = column cu, a = column ca, q = column cq)
  auto wdot3 = [&](int cu, int ca, int cq, bool three, float& suu, float& sua, float& sqa) {
    const float* u = sp + cu * LD;
    const float* a = sp + ca * LD;
    const float* q = sp + cq * LD;
    float s0 = 0.f, s1 = 0.f, s2 = 0.f;
    for (int i = c_lo + lane; i < c_hi; i += 32) {
      const float uv = u[i];
      s0 = fmaf(uv, uv, s0);
      if (three) {
        const float av = a[i];
        s1 = fmaf(uv, av, s1);
        s2 = fmaf(q[i], av, s2);
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      s0 += __shfl_xor_sync(0xffffffffu, s0, o);
      s1 += __shfl_xor_sync(0xffffffffu, s1, o);
      s2 += __shfl_xor_sync(0xffffffffu, s2, o);
    }
    suu = s0;
    sua = s1;
    sqa = s2;
  };
  // round tags of the tagged exchange: unique per (launch, round)
  // Fixed-point exchange (rounds t >= 1, xmode 2): value k of round t is scaled by 2^e
  // with e chosen from a bound on |partial| (column norms of round 0), rounded to an
  // integer |v| <= 2^46 and added with ONE red.add.u64 per CTA to word W[t&1][k] as
  //     (1 << 56) + (v + 2^46)          -- top byte counts arrivals, low 56 bits sum
  // Integer addition is associative, so the total is independent of arrival order
  // (deterministic) and exact in fixed point; the word is never reset within a launch:
  // readers take the difference with the value they saw two rounds earlier.
  auto fx_exp = [&](int t, int k) -> int {
    // |partial| <= bound: 4||a_t||^2, 4||a_t|| ||a_{t+1}||, 4||a_{t+1}||, 4||a_{t+2}|| for value
    // classes 0, 1, 2, 3+ (u_t shrinks a_t, ||q_i|| <= 1); 2||a_j|| < 2^exS[j]
    if (k == 0) return FX_VBITS - 2 * exS[t];
    if (k == 1) return FX_VBITS - (exS[t] + exS[t + 1]);
    if (k == 2) return FX_VBITS - (exS[t + 1] + 1);
    return FX_VBITS - (exS[t + 2] + 1);
  };
  // publish the L values of part[][] as this CTA's partial vector of round t, arrive
  auto publish_arrive = [&](int t, int L) {
    __syncthreads();
    const bool fx = p.xmode == 2 && t > 0;
    float* buf = p.partials + (size_t)(t & 1) * (LEAF_MAX_W + 2) * G;
    // sum of the GEMV_PARTS row-part partials of value k: 4 threads per value, each
    // adds a quarter of the parts, then a 2-level xor tree (fixed order)
    const int k = threadIdx.x >> 2, jq = threadIdx.x & 3;
    float s = 0.f;
    if (k < L) {
#pragma unroll
      for (int q = 0; q < GEMV_PARTS / 4; ++q) s += part[t & 1][jq * (GEMV_PARTS / 4) + q][k];
    }
    s += __shfl_xor_sync(0xffffffffu, s, 1);
    s += __shfl_xor_sync(0xffffffffu, s, 2);
    if (k < L && jq == 0) {
      if (fx) {
        long long v = __double2ll_rn((double)s * pow2d(fx_exp(t, k)));
        const long long vb = 1ll << FX_VBITS;
        v = v > vb ? vb : (v < -vb ? -vb : v);
        const unsigned long long add = (1ull << FX_CNT_SHIFT) + (unsigned long long)(v + vb);
        const size_t off = ((size_t)(t & 1) * (LEAF_MAX_W + 2) + k) * LEAF_XW_COPIES + g % LEAF_XW_COPIES;
        if (!p.sys) {
          asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p.xw + off), "l"(add) : "memory");
        } else {
          // row-sharded run: the same word on every GPU receives every CTA's partial
          for (int j = 0; j < p.nranks; ++j)
            asm volatile("red.relaxed.sys.global.add.u64 [%0], %1;" ::"l"(p.xw_peers[j] + off), "l"(add)
                         : "memory");
        }
      } else {
        buf[(size_t)k * G + g] = s;
      }
    }
    if (!fx) {
      __syncthreads();
      if (threadIdx.x == 0)  // release: orders this CTA's partial stores (bar.sync cumulativity)
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(p.counter) : "memory");
    }
  };

  // Round layout (t >= 1), R19:  [0] u_t.u_t  [1] u_t.a_{t+1}  [2] q_{t-1}.a_{t+1}
  // [3+i] q_i.a_{t+2} (i <= t-1).  The q_i.a_{t+2} values are published one round ahead, so
  // after round t every CTA already knows r_{i,t+2} (i <= t-1) and can subtract those
  // projections from a_{t+2} while round t+1's exchange is in flight; after that exchange
  // only q_t and q_{t+1} remain to be subtracted (two columns on the critical path).
  auto round_len = [&](int t) -> int {
    if (t == 0) return w + (w > 1 ? 1 : 0);
    if (t == w - 1) return 1;
    if (t == w - 2) return 3;
    return t + 3;
  };
  // col -= sum_{i < cnt} q_i * cf[i]   (4 rows per thread, fixed order of i within two sums)
  auto project_out = [&](int col, int cnt, const float* cf) {
    float* an = sp + col * LD;
    for (int v = threadIdx.x; v < nv4; v += LEAF_THREADS) {
      float4 a0 = make_float4(0.f, 0.f, 0.f, 0.f), a1 = a0;
      int k = 0;
      for (; k + 4 <= cnt; k += 4) {
        const float4 c = reinterpret_cast<const float4*>(cf)[k >> 2];
        const float4 x0 = reinterpret_cast<const float4*>(sp + (k + 0) * LD)[v];
        const float4 x1 = reinterpret_cast<const float4*>(sp + (k + 1) * LD)[v];
        const float4 x2 = reinterpret_cast<const float4*>(sp + (k + 2) * LD)[v];
        const float4 x3 = reinterpret_cast<const float4*>(sp + (k + 3) * LD)[v];
        a0.x = fmaf(x0.x, c.x, a0.x); a0.y = fmaf(x0.y, c.x, a0.y); a0.z = fmaf(x0.z, c.x, a0.z); a0.w = fmaf(x0.w, c.x, a0.w);
        a1.x = fmaf(x1.x, c.y, a1.x); a1.y = fmaf(x1.y, c.y, a1.y); a1.z = fmaf(x1.z, c.y, a1.z); a1.w = fmaf(x1.w, c.y, a1.w);
        a0.x = fmaf(x2.x, c.z, a0.x); a0.y = fmaf(x2.y, c.z, a0.y); a0.z = fmaf(x2.z, c.z, a0.z); a0.w = fmaf(x2.w, c.z, a0.w);
        a1.x = fmaf(x3.x, c.w, a1.x); a1.y = fmaf(x3.y, c.w, a1.y); a1.z = fmaf(x3.z, c.w, a1.z); a1.w = fmaf(x3.w, c.w, a1.w);
      }
      for (; k < cnt; ++k) {
        const float c = cf[k];
        const float4 x = reinterpret_cast<const float4*>(sp + k * LD)[v];
        a0.x = fmaf(x.x, c, a0.x); a0.y = fmaf(x.y, c, a0.y); a0.z = fmaf(x.z, c, a0.z); a0.w = fmaf(x.w, c, a0.w);
      }
      float4 av = reinterpret_cast<float4*>(an)[v];
      av.x -= a0.x + a1.x;
      av.y -= a0.y + a1.y;
      av.z -= a0.z + a1.z;
      av.w -= a0.w + a1.w;
      reinterpret_cast<float4*>(an)[v] = av;
    }
  };

  // ---- round 0 vector: [ ||a_k||^2 (k < w), a_0^T a_1 ] ----
  // (r0_mode 2: the globally reduced round-0 vector is given in p.r0buf)
  if (p.r0_mode != 2) {
    const int t = 0;
    const int L = round_len(0);
    DBG_STAMP(0);
    for (int k = kq; k < L; k += 32) {
      int cx, cy;
      round_operands(0, w, k, cx, cy);
      part[0][warp][k] = dot4(cx, cy);
    }
    publish_arrive(0, L);
  }

  for (int t = 0; t < w; ++t) {
    const int L = round_len(t);
    const bool fx = p.xmode == 2 && t > 0;
    const bool given = t == 0 && p.r0_mode == 2;
    // ---- wait for round t (counter barrier for round 0 / xmode 0) ----
    if (!fx && !given && threadIdx.x == 0) {
      unsigned cv;
      const unsigned target = (p.xmode == 2 ? 1u : (unsigned)(t + 1)) * (unsigned)G;
      do {
        asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(cv) : "l"(p.counter) : "memory");
      } while (cv < target);
    }
    __syncthreads();
    if (fx) {
      // ---- fixed-point exchange: each value's word is polled by its thread until all
      //      ranks x G CTAs have added ----
      // LEAF_XW_COPIES threads per value, one word copy each; the copies' integer totals are
      // summed with an xor tree (exact, so the order does not matter)
      const int k = threadIdx.x / LEAF_XW_COPIES, hc = threadIdx.x % LEAF_XW_COPIES;
      long long total = 0;
      if (k < L) {
        const int widx = ((t & 1) * (LEAF_MAX_W + 2) + k) * LEAF_XW_COPIES + hc;
        const unsigned cnt_h =
            (unsigned)p.nranks * (unsigned)(G / LEAF_XW_COPIES + (hc < G % LEAF_XW_COPIES ? 1 : 0));
        const unsigned long long* wp = p.xw + widx;
        const unsigned long long prev = xprev[widx];
        unsigned long long now = ld_word(wp, p.sys), d = now - prev;
        long long spins = 0;
        while ((unsigned)(d >> FX_CNT_SHIFT) != cnt_h) {
          now = ld_word(wp, p.sys);
          d = now - prev;
          if (++spins > (1ll << 27)) {            // ~seconds: a peer is missing -- fail, never hang
            atomicExch(p.breakdown, -2);
            break;
          }
        }
        xprev[widx] = now;
        total = (long long)(d & ((1ull << FX_CNT_SHIFT) - 1)) - (long long)cnt_h * (1ll << FX_VBITS);
      }
#pragma unroll
      for (int o = 1; o < LEAF_XW_COPIES; o <<= 1) total += __shfl_xor_sync(0xffffffffu, total, o);
      if (k < L && hc == 0) {
        const float val = (float)((double)total * pow2d(-fx_exp(t, k)));
        tot[k] = val;
        if (k >= 3) coef[t & 1][k - 3] = val;
      }
    } else if (given) {
      if (threadIdx.x < L) {
        const int k = threadIdx.x;
        const float s = p.r0buf[k];
        tot[k] = s;
        if (k < w) {
          anorm2[k] = s;
          int ex;
          frexpf(2.0f * sqrtf(s), &ex);
          exS[k] = ex;
          tauc[k] = (float)p.m_global * u_work * sqrtf(s);
        }
      }
    } else {
      // ---- gather round t's G partials per value, fixed-order sum ----
      constexpr int KPW = (LEAF_MAX_W + 2 + LEAF_WARPS - 1) / LEAF_WARPS;
      constexpr int QMAX = (LEAF_MAX_G + 31) / 32;
      const float* buf = p.partials + (size_t)(t & 1) * (LEAF_MAX_W + 2) * G;
      float v[KPW][QMAX];
#pragma unroll
      for (int a = 0; a < KPW; ++a)
#pragma unroll
        for (int q = 0; q < QMAX; ++q) {
          const int k = warp + a * LEAF_WARPS, c = lane + 32 * q;
          v[a][q] = (k < L && c < G) ? __ldcg(buf + (size_t)k * G + c) : 0.0f;
        }
#pragma unroll
      for (int a = 0; a < KPW; ++a) {
        const int k = warp + a * LEAF_WARPS;
        if (k >= L) break;                               // warp-uniform
        float s = v[a][0];
#pragma unroll
        for (int q = 1; q < QMAX; ++q) s += v[a][q];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
        if (lane == 0) {
          tot[k] = s;
          if (t > 0 && k >= 3) coef[t & 1][k - 3] = s;
          if (t == 0 && k < w) {
            anorm2[k] = s;
            int ex;
            frexpf(2.0f * sqrtf(s), &ex);
            exS[k] = ex;
            tauc[k] = (float)p.m_global * u_work * sqrtf(s);
          }
        }
      }
    }
    __syncthreads();
    DBG_STAMP(2);
    if (t == 0 && p.r0_mode == 1) {
      // round-0-only launch of a row-sharded run: hand the local vector to the host
      // (which all-reduces it across GPUs) and stop
      if (g == 0 && threadIdx.x < L) p.r0buf[threadIdx.x] = tot[threadIdx.x];
      return;
    }
    // ---- scalars (every thread, identical): r_tt, 1/r_tt, r_{t,t+1}, r_{t-1,t+1} ----
    const bool more = t + 1 < w;
    const float uu = tot[0];
    const float ua = (t == 0) ? ((w > 1) ? tot[w] : 0.0f) : (more ? tot[1] : 0.0f);
    const float cq = (t >= 1 && more) ? tot[2] : 0.0f;   // r_{t-1,t+1} = q_{t-1}^T a_{t+1}
    float rtt = sqrtf(uu);
    const float tau = tauc[t];
    const bool bad = !(rtt > tau) || !isfinite(rtt);
    const float inv = bad ? 0.0f : 1.0f / rtt;
    if (bad) rtt = 0.0f;
    const float ct = ua * inv;                            // r_{t,t+1}
    if (g == 0) {
      if (threadIdx.x == 0) {
        p.R[t + (int64_t)t * p.ldr] = rtt;
        if (bad) atomicMin(p.breakdown, (int)(p.col_offset + t));
      }
      if (more && threadIdx.x <= t) {
        const int i = threadIdx.x;
        const float r = (i == t) ? ct : (i == t - 1) ? cq : coef[(t - 1) & 1][i];   // i <= t-2: round t-1
        p.R[i + (int64_t)(t + 1) * p.ldr] = r;
      }
      if (threadIdx.x > t && threadIdx.x < w) p.R[threadIdx.x + (int64_t)t * p.ldr] = 0.0f;
    }
    DBG_STAMP(5);
    // ---- q_t = u_t / r_tt (stored rounded); u_{t+1} = w_{t+1} - q_{t-1} r_{t-1,t+1} - q_t r_{t,t+1}
    //      where w_{t+1} = a_{t+1} - sum_{i<=t-2} q_i r_{i,t+1} was formed during round t ----
    {
      float* ut = sp + t * LD;
      float* an = sp + (t + 1) * LD;
      const float* qp = sp + (t >= 1 ? t - 1 : 0) * LD;
      for (int v = threadIdx.x; v < ((p.skip & 1) ? 0 : nv4); v += LEAF_THREADS) {
        float4 q4 = reinterpret_cast<float4*>(ut)[v];
        q4.x *= inv; q4.y *= inv; q4.z *= inv; q4.w *= inv;
        reinterpret_cast<float4*>(ut)[v] = q4;
        {
          const int i0 = 4 * v;
          T* dst = P + r0 + i0 + (int64_t)t * p.ldp;
          if (p.vec_ok && i0 + 4 <= rows) {
            store4<T>(dst, q4);
          } else {
            const float qv[4] = {q4.x, q4.y, q4.z, q4.w};
            for (int e = 0; e < 4 && i0 + e < rows; ++e) dst[e] = Elem<T>::store(qv[e]);
          }
        }
        if (more) {
          float4 av = reinterpret_cast<float4*>(an)[v];
          if (t >= 1) {
            const float4 qm = reinterpret_cast<const float4*>(qp)[v];
            av.x = fmaf(-qm.x, cq, av.x); av.y = fmaf(-qm.y, cq, av.y);
            av.z = fmaf(-qm.z, cq, av.z); av.w = fmaf(-qm.w, cq, av.w);
          }
          av.x = fmaf(-q4.x, ct, av.x); av.y = fmaf(-q4.y, ct, av.y);
          av.z = fmaf(-q4.z, ct, av.z); av.w = fmaf(-q4.w, ct, av.w);
          reinterpret_cast<float4*>(an)[v] = av;
        }
      }
    }
    __syncthreads();
    DBG_STAMP(4);
    if (!more) break;
    // ---- round t+1: the dots that needed round t -- u_{t+1}.u_{t+1}, u_{t+1}.a_{t+2},
    //      q_t.a_{t+2}, q_t.a_{t+3} -- then publish + arrive ----
    {
      const int t1 = t + 1;
      const int L1 = round_len(t1);
      if (p.dbg != nullptr && blockIdx.x == DBG_CTA && threadIdx.x == 0) p.dbg[(size_t)t1 * 8] = clock64();
      const bool h2 = t + 2 < w, h3 = t + 3 < w;
      const float* u = sp + t1 * LD;
      const float* qv = sp + t * LD;
      const float* a2 = sp + (h2 ? t + 2 : t1) * LD;
      const float* a3 = sp + (h3 ? t + 3 : t1) * LD;
      float s0 = 0.f, s1 = 0.f, s2 = 0.f, s3 = 0.f;
      if (!(p.skip & 4)) {
        for (int i = c_lo + lane; i < c_hi; i += 32) {
          const float uv = u[i];
          s0 = fmaf(uv, uv, s0);
          if (h2) {
            const float av = a2[i], qq = qv[i];
            s1 = fmaf(uv, av, s1);
            s2 = fmaf(qq, av, s2);
            if (h3) s3 = fmaf(qq, a3[i], s3);
          }
        }
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        s0 += __shfl_xor_sync(0xffffffffu, s0, o);
        s1 += __shfl_xor_sync(0xffffffffu, s1, o);
        s2 += __shfl_xor_sync(0xffffffffu, s2, o);
        s3 += __shfl_xor_sync(0xffffffffu, s3, o);
      }
      if (p.dbg != nullptr && blockIdx.x == DBG_CTA && threadIdx.x == 0) p.dbg[(size_t)t1 * 8 + 6] = clock64();
      if (lane == 0) {
        float* pw = part[t1 & 1][warp];
        pw[0] = s0;
        if (h2) {
          pw[1] = s1;
          pw[2] = s2;
          if (h3) pw[3 + t] = s3;                        // q_t.a_{t1+2}: index 3 + (t1 - 1)
        }
      }
      publish_arrive(t1, L1);
      if (p.dbg != nullptr && blockIdx.x == DBG_CTA && threadIdx.x == 0) p.dbg[(size_t)t1 * 8 + 7] = clock64();
    }
    // ---- while round t+1's exchange is in flight:
    //      (a) lookahead for round t+2: q_i.a_{t+4}, i <= t  (index 3 + i)
    //      (b) w_{t+2} = a_{t+2} - sum_{i <= t-1} q_i r_{i,t+2}  (coefficients from round t) ----
    if (t + 4 < w && !(p.skip & 2)) {
      const int cnt = t + 1;                              // i in [0, t]
      const bool ha = kq < cnt, hb = kq + 32 < cnt;
      if (ha) {
        const float4* y = reinterpret_cast<const float4*>(sp + (t + 4) * LD);
        const float4* xa = reinterpret_cast<const float4*>(sp + kq * LD);
        const float4* xb = reinterpret_cast<const float4*>(sp + (hb ? kq + 32 : kq) * LD);
        float a0 = 0.f, a1 = 0.f, b0 = 0.f, b1 = 0.f;
        for (int i = v_lo; i < v_hi; ++i) {
          const float4 yy = y[i], a = xa[i];
          a0 = fmaf(a.x, yy.x, a0);
          a1 = fmaf(a.y, yy.y, a1);
          a0 = fmaf(a.z, yy.z, a0);
          a1 = fmaf(a.w, yy.w, a1);
          if (hb) {
            const float4 b = xb[i];
            b0 = fmaf(b.x, yy.x, b0);
            b1 = fmaf(b.y, yy.y, b1);
            b0 = fmaf(b.z, yy.z, b0);
            b1 = fmaf(b.w, yy.w, b1);
          }
        }
        float* pw = part[t & 1][warp];                    // round t+2 has the parity of t
        pw[3 + kq] = a0 + a1;
        if (hb) pw[3 + kq + 32] = b0 + b1;
      }
    }
    if (t + 2 < w && t >= 1) project_out(t + 2, t, coef[t & 1]);
    if (p.dbg != nullptr && blockIdx.x == DBG_CTA && threadIdx.x == 0) p.dbg[(size_t)(t + 1) * 8 + 1] = clock64();
  }
  // every CTA ends with the same last-seen words; CTA 0 persists them for the next launch
  if (g == 0)
    for (int i = threadIdx.x; i < LEAF_XW_WORDS; i += blockDim.x) p.xprev_g[i] = xprev[i];
}

template <typename T>
cudaError_t launch_leaf(const LeafParams& p, int grid, cudaStream_t st) {
  const size_t smem = (size_t)p.w * leaf_ld(p.rows_per_cta) * sizeof(float);
  static size_t attr_smem = 0;
  if (smem > attr_smem) {
    cudaError_t e = cudaFuncSetAttribute(leaf_cgs_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)smem);
    if (e != cudaSuccess) return e;
    attr_smem = smem;
  }
  cudaError_t e = cudaMemsetAsync(p.counter, 0, sizeof(unsigned int), st);
  if (e != cudaSuccess) return e;
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
  return cudaLaunchKernelEx(&cfg, leaf_cgs_kernel<T>, p);
}

int leaf_max_smem_rows(int w) { return (int)((LEAF_SMEM_BUDGET) / ((size_t)w * sizeof(float))); }

template cudaError_t launch_leaf<__half>(const LeafParams&, int, cudaStream_t);
template cudaError_t launch_leaf<__nv_bfloat16>(const LeafParams&, int, cudaStream_t);
template cudaError_t launch_leaf<float>(const LeafParams&, int, cudaStream_t);

}  // namespace rgsqr
