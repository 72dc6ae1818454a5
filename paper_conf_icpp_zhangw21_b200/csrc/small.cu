// small.cu -- the bottom nodes of the recursion (Eq. 2) in one kernel:
//     R12 = Q1^T A2        (inner product, w1 x w2, both <= 64)
//     A2 <- A2 - Q1 R12    (outer product, fused subtraction, rounded once to storage)
// for fp16 / bf16 storage.  Separately these are a split-K TN GEMM, a split-K reduction and
// an NN GEMM -- three launches that each re-read the m x 64 operands; at the bottom of the
// recursion they are bound by HBM bytes and launch latency, not by the tensor cores.
//
// Cooperative grid, one CTA per SM, CTA g owns rows [g RP, (g+1) RP):
//   phase 1: the CTA's row slices of Q1 and A2 are loaded ONCE into shared memory; the partial
//            Q1_s^T A2_s (64 x 64, fp32) is formed with mma.sync m16n8k16 and written out;
//   barrier; phase 2: every CTA sums 1/G of the entries over all G partials in a fixed
//            order (deterministic) -> R12 (fp32, the R block) and its operand copy (RN);
//   barrier; phase 3: A2_s -= Q1_s R12 with mma.sync from the same shared-memory slices;
//            A2' rounded RN and stored once.
// Reads Q1 and A2 once and writes A2 once (plus 2 x G x 16 KB of partials in L2).
#include "dtype.cuh"
#include "kernels.h"

namespace rgsqr {

static constexpr int SN_THREADS = 256;

// W: the widest w1 / w2 the instance handles (64 or 128).  A2 is processed in NH = W / 64
// column halves of 64, so the slices fit shared memory; R12 is W x W.
template <int W>
struct SNCfg {
  static constexpr int NH = W / 64;
  static constexpr int RS = W + 8;       // R12 operand tile stride (halves): 2 RS == 16 (mod 128)
  static constexpr int E = W * W;        // R12 entries
  static constexpr int MT = W / 16;      // m-tiles of R12 in phase 1 (= n-tiles per warp)
};

// shared-memory column stride (halves) of a row slice: >= rows rounded to 16, and
// 2 * stride == 16 (mod 128) bytes so that ldmatrix row addresses hit distinct banks
__host__ __device__ inline int sn_stride(int rp) {
  const int r16 = (rp + 15) & ~15;
  return r16 + ((8 - (r16 % 64)) + 64) % 64;
}

size_t small_node_smem(int rp, int w) {
  return (size_t)(w + 64) * sn_stride(rp) * 2 + (size_t)64 * (w + 8) * 2 + 8 * 65 * 4 + 64;
}

template <typename T>
struct MmaOp;
template <>
struct MmaOp<__half> {
  __device__ static void mma(float* d, const uint32_t* a, const uint32_t* b) {
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
  }
};
template <>
struct MmaOp<__nv_bfloat16> {
  __device__ static void mma(float* d, const uint32_t* a, const uint32_t* b) {
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
  }
};

__device__ __forceinline__ void ldsm_x4(uint32_t* r, const void* p) {
  const unsigned a = (unsigned)__cvta_generic_to_shared(p);
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3])
               : "r"(a));
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t* r, const void* p) {
  const unsigned a = (unsigned)__cvta_generic_to_shared(p);
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3])
               : "r"(a));
}

// grid barrier on a never-reset counter: release this CTA's writes, wait until the counter reaches
// `target` (wrap-safe), acquire all
__device__ __forceinline__ void sn_grid_barrier(unsigned* counter, unsigned target) {
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(counter) : "memory");
    unsigned v;
    do {
      asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(counter) : "memory");
    } while ((int)(v - target) < 0);
  }
  __syncthreads();
}

// columns [c0, c0 + ncols) of a column-major m x * operand, rows [r0, r0 + rows), into a
// [ncols_alloc][S] shared slice (zero-padded): cp.async 16-byte copies + scalar tail
template <typename T>
__device__ __forceinline__ void sn_load_cols(T* dst, int S, const T* src, int64_t ld, int64_t r0, int rows, int c0,
                                             int ncols, int ncols_alloc, bool vec_ok) {
  const int nv = vec_ok ? rows / 8 : 0;
  for (int idx = threadIdx.x; idx < ncols_alloc * (S / 8); idx += SN_THREADS) {
    const int c = idx / (S / 8), v = idx - c * (S / 8);
    const bool in = v < nv && c < ncols;
    const T* sp = in ? src + r0 + 8 * v + (int64_t)(c0 + c) * ld : src;
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"((unsigned)__cvta_generic_to_shared(dst + c * S + 8 * v)),
                 "l"(sp), "r"(in ? 16 : 0)
                 : "memory");
  }
  asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
  __syncthreads();
  const int tl = rows - 8 * nv;
  for (int idx = threadIdx.x; idx < ncols * tl; idx += SN_THREADS) {
    const int c = idx / tl, r = 8 * nv + (idx - c * tl);
    dst[c * S + r] = src[r0 + r + (int64_t)(c0 + c) * ld];
  }
  __syncthreads();
}

template <typename T, int W>
__global__ void __launch_bounds__(SN_THREADS, 1) small_node_kernel(SmallNodeParams p) {
  using C = SNCfg<W>;
  extern __shared__ __align__(16) unsigned char smem[];
  const int RP = p.rows_per_cta;
  const int S = sn_stride(RP);
  const int RP16 = (RP + 15) & ~15;
  T* qs = reinterpret_cast<T*>(smem);            // [W][S]: column i of the Q1 slice
  T* as = qs + W * S;                            // [64][S]: column j of the current A2 half
  T* rs = as + 64 * S;                           // [64][RS]: R12 operand of the half as [j][i]
  float* red = reinterpret_cast<float*>(rs + 64 * C::RS);   // [8][33] phase 2, [8][65] phase 3
  const int G = gridDim.x, g = blockIdx.x;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int q = lane >> 3, l8 = lane & 7;
  const int64_t r0 = (int64_t)g * RP;
  const int64_t rem = p.m - r0;
  const int rows = rem <= 0 ? 0 : (rem < RP ? (int)rem : RP);
  const T* Q1 = static_cast<const T*>(p.Q1);
  T* A2 = static_cast<T*>(p.A2);
  const bool vec = p.vec_ok != 0;

  // ---- phase 1: partial = Q1_s^T A2_s (W x W); per A2 half: warp = m-tile warp % MT,
  //      n-tiles (warp / MT) * MT .. + MT - 1 of the half ----
  sn_load_cols(qs, S, Q1, p.ldq, r0, rows, 0, p.w1, W, vec);
  float* P = p.partials + (size_t)g * C::E;      // [j][i], i contiguous
  for (int hh = 0; hh < C::NH; ++hh) {
    sn_load_cols(as, S, static_cast<const T*>(A2), p.lda, r0, rows, 64 * hh, max(0, min(64, p.w2 - 64 * hh)), 64, vec);
    const int mt = warp % C::MT, nt0 = (warp / C::MT) * C::MT;
    float acc[C::MT][4] = {};
    for (int kk = 0; kk < RP16; kk += 16) {
      uint32_t a[4], b[C::MT / 2][4];
      ldsm_x4(a, qs + (16 * mt + (q & 1) * 8 + l8) * S + kk + (q >> 1) * 8);
#pragma unroll
      for (int h = 0; h < C::MT / 2; ++h)
        ldsm_x4(b[h], as + (8 * (nt0 + 2 * h + (q >> 1)) + l8) * S + kk + (q & 1) * 8);
#pragma unroll
      for (int n = 0; n < C::MT; ++n) MmaOp<T>::mma(acc[n], a, &b[n >> 1][(n & 1) * 2]);
    }
#pragma unroll
    for (int n = 0; n < C::MT; ++n) {
      const int i = 16 * mt + (lane >> 2), j = 64 * hh + 8 * (nt0 + n) + 2 * (lane & 3);
      P[j * W + i] = acc[n][0];
      P[(j + 1) * W + i] = acc[n][1];
      P[j * W + i + 8] = acc[n][2];
      P[(j + 1) * W + i + 8] = acc[n][3];
    }
    __syncthreads();                               // before the next half overwrites `as`
  }
  sn_grid_barrier(p.counter, p.counter_base + (unsigned)G);

  // ---- phase 2: entries [g EPC, (g+1) EPC) summed over the G partials in a fixed order:
  //      warp k adds partials k, k+8, ... in order, then warp 0 the 8 groups ----
  {
    const int EPC = (C::E + G - 1) / G;
    const int e_end = min(C::E, (g + 1) * EPC);
    for (int e0 = g * EPC; e0 < e_end; e0 += 32) {
      const int e = e0 + lane;
      const bool ok = e < e_end;
      // all of this thread's partials in flight at once, then summed in order
      constexpr int PMAX = (LEAF_MAX_G + 7) / 8;
      float v[PMAX];
#pragma unroll
      for (int qq = 0; qq < PMAX; ++qq) {
        const int k = warp + 8 * qq;
        v[qq] = (ok && k < G) ? __ldcg(p.partials + (size_t)k * C::E + e) : 0.0f;
      }
      float s0 = v[0];
#pragma unroll
      for (int qq = 1; qq < PMAX; ++qq) s0 += v[qq];
      red[warp * 33 + lane] = s0;
      __syncthreads();
      if (warp == 0 && ok) {
        float vv = red[lane];
#pragma unroll
        for (int k = 1; k < 8; ++k) vv += red[k * 33 + lane];
        const int i = e % W, j = e / W;
        if (i < p.w1 && j < p.w2) p.R12[i + (int64_t)j * p.ldr] = vv;
        static_cast<T*>(p.r12op)[e] = Elem<T>::store(vv);   // [j][i]; zero outside w1 x w2
      }
      __syncthreads();
    }
  }
  sn_grid_barrier(p.counter, p.counter_base + (unsigned)(2 * G));

  // ---- phase 3: A2_s -= Q1_s R12 per half; warp: m-tiles warp, warp + 8, ... (16 rows), all
  //      8 n-tiles of the half, K = W ----
  for (int hh = 0; hh < C::NH; ++hh) {
    const int nc = max(0, min(64, p.w2 - 64 * hh));   // valid columns of this half
    if (C::NH > 1)
      sn_load_cols(as, S, static_cast<const T*>(A2), p.lda, r0, rows, 64 * hh, nc, 64, vec);
    for (int idx = threadIdx.x; idx < 64 * (W / 8); idx += SN_THREADS) {   // 64 x W halves, 16 B each
      const int j = idx / (W / 8), v = idx - j * (W / 8);
      *reinterpret_cast<uint4*>(rs + j * C::RS + 8 * v) =
          __ldcg(reinterpret_cast<const uint4*>(static_cast<const T*>(p.r12op) + (size_t)(64 * hh + j) * W + 8 * v));
    }
    __syncthreads();
    // the next leaf's round 0 (leaf r0_mode 3, W == 64): squares of the ROUNDED A2' values per
    // column (and a_0.a_1), accumulated from the epilogue registers, reduced in a fixed order below
    float nrm[8][2] = {};
    float d01 = 0.f;
    for (int mt = warp; mt < RP16 / 16; mt += SN_THREADS / 32) {
      float acc[8][4] = {};
#pragma unroll
      for (int ks = 0; ks < W / 16; ++ks) {
        uint32_t a[4], b[4][4];
        // A[m = row][k = i] lives as qs[i][row]: transposed 8x8 loads
        ldsm_x4_t(a, qs + (16 * ks + (q >> 1) * 8 + l8) * S + 16 * mt + (q & 1) * 8);
#pragma unroll
        for (int h = 0; h < 4; ++h) ldsm_x4(b[h], rs + (8 * (2 * h + (q >> 1)) + l8) * C::RS + 16 * ks + (q & 1) * 8);
#pragma unroll
        for (int n = 0; n < 8; ++n) MmaOp<T>::mma(acc[n], a, &b[n >> 1][(n & 1) * 2]);
      }
#pragma unroll
      for (int n = 0; n < 8; ++n) {
        const int r = 16 * mt + (lane >> 2), j = 8 * n + 2 * (lane & 3);
        T* c0 = as + j * S + r;
        T* c1 = as + (j + 1) * S + r;
        const T v00 = Elem<T>::store(Elem<T>::load(c0[0]) - acc[n][0]);
        const T v01 = Elem<T>::store(Elem<T>::load(c1[0]) - acc[n][1]);
        const T v10 = Elem<T>::store(Elem<T>::load(c0[8]) - acc[n][2]);
        const T v11 = Elem<T>::store(Elem<T>::load(c1[8]) - acc[n][3]);
        c0[0] = v00;
        c1[0] = v01;
        c0[8] = v10;
        c1[8] = v11;
        if (W == 64) {
          const float f00 = Elem<T>::load(v00), f01 = Elem<T>::load(v01), f10 = Elem<T>::load(v10),
                      f11 = Elem<T>::load(v11);
          nrm[n][0] = fmaf(f00, f00, fmaf(f10, f10, nrm[n][0]));
          nrm[n][1] = fmaf(f01, f01, fmaf(f11, f11, nrm[n][1]));
          if (n == 0) d01 = fmaf(f00, f01, fmaf(f10, f11, d01));   // columns 0, 1 on lanes with tig 0
        }
      }
    }
    const bool r0w = W == 64 && p.r0_partials != nullptr;
    if (r0w) {
      // lanes sharing tig (= lane & 3) hold the same columns: xor tree over the row groups
#pragma unroll
      for (int n = 0; n < 8; ++n)
#pragma unroll
        for (int c = 0; c < 2; ++c) {
          float v = nrm[n][c];
          v += __shfl_xor_sync(0xffffffffu, v, 4);
          v += __shfl_xor_sync(0xffffffffu, v, 8);
          v += __shfl_xor_sync(0xffffffffu, v, 16);
          nrm[n][c] = v;
        }
      d01 += __shfl_xor_sync(0xffffffffu, d01, 4);
      d01 += __shfl_xor_sync(0xffffffffu, d01, 8);
      d01 += __shfl_xor_sync(0xffffffffu, d01, 16);
      if (lane < 4) {
#pragma unroll
        for (int n = 0; n < 8; ++n) {
          red[warp * 65 + 8 * n + 2 * lane] = nrm[n][0];
          red[warp * 65 + 8 * n + 2 * lane + 1] = nrm[n][1];
        }
        if (lane == 0) red[warp * 65 + 64] = d01;
      }
    }
    __syncthreads();
    if (r0w) {
      const int L = p.w2 + (p.w2 > 1 ? 1 : 0);
      for (int k = threadIdx.x; k < L; k += SN_THREADS) {
        const int col = k < p.w2 ? k : 64;
        float v = red[col];
#pragma unroll
        for (int wv = 1; wv < SN_THREADS / 32; ++wv) v += red[wv * 65 + col];
        p.r0_partials[(size_t)k * G + g] = v;
      }
    }
    // ---- store A2' of this half (valid columns, rows < rows) ----
    const int nv = vec ? rows / 8 : 0;
    for (int idx = threadIdx.x; idx < nc * nv; idx += SN_THREADS) {
      const int c = idx / nv, v = idx - c * nv;
      *reinterpret_cast<uint4*>(A2 + r0 + 8 * v + (int64_t)(64 * hh + c) * p.lda) =
          *reinterpret_cast<const uint4*>(as + c * S + 8 * v);
    }
    const int tl = rows - 8 * nv;
    for (int idx = threadIdx.x; idx < nc * tl; idx += SN_THREADS) {
      const int c = idx / tl, r = 8 * nv + (idx - c * tl);
      A2[r0 + r + (int64_t)(64 * hh + c) * p.lda] = as[c * S + r];
    }
    __syncthreads();                               // before the next half overwrites `as`, `rs`
  }
}

template <typename T, int W>
static cudaError_t launch_small_node_w(const SmallNodeParams& p, int grid, cudaStream_t st) {
  const size_t smem = small_node_smem(p.rows_per_cta, W);
  static size_t attr = 0;
  if (smem > attr) {
    cudaError_t e = cudaFuncSetAttribute(small_node_kernel<T, W>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr = smem;
  }
  SmallNodeParams q = p;   // two barriers per launch on the never-reset counter
  q.counter_base = *p.counter_host;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(SN_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr1[1];
  attr1[0].id = cudaLaunchAttributeCooperative;
  attr1[0].val.cooperative = 1;
  cfg.attrs = attr1;
  cfg.numAttrs = 1;
  cudaError_t e = cudaLaunchKernelEx(&cfg, small_node_kernel<T, W>, q);
  if (e == cudaSuccess) *p.counter_host += 2u * (unsigned)grid;   // (only launched arrivals count)
  return e;
}

template <typename T>
cudaError_t launch_small_node(const SmallNodeParams& p, int grid, cudaStream_t st) {
  if (p.w1 <= 64 && p.w2 <= 64) return launch_small_node_w<T, 64>(p, grid, st);
  return launch_small_node_w<T, 128>(p, grid, st);
}

template cudaError_t launch_small_node<__half>(const SmallNodeParams&, int, cudaStream_t);
template cudaError_t launch_small_node<__nv_bfloat16>(const SmallNodeParams&, int, cudaStream_t);

}  // namespace rgsqr
