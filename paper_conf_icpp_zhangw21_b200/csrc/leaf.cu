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
// (reading R19).  A round = per-warp partial dot products over the CTA's
// rows, one partial vector per CTA to global memory, a grid barrier (release/acquire
// counter), then every CTA sums the G partials in the same fixed order (deterministic,
// no float atomics).
#include <cooperative_groups.h>

#include "dtype.cuh"
#include "kernels.h"

namespace rgsqr {

static constexpr int LEAF_THREADS = 256;
static constexpr int LEAF_WARPS = LEAF_THREADS / 32;

__device__ __forceinline__ void grid_barrier(unsigned int* counter, unsigned int target) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(counter, 1u);
    unsigned int v;
    do {
      asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(counter) : "memory");
    } while (v < target);
    __threadfence();
  }
  __syncthreads();
}

template <typename T>
__global__ void __launch_bounds__(LEAF_THREADS, 1) leaf_cgs_kernel(LeafParams p) {
  extern __shared__ float sp[];                     // [w][RP] column-major panel slice
  __shared__ float tot[LEAF_MAX_W + 2];            // reduced round vector
  __shared__ float anorm2[LEAF_MAX_W];             // ||a_k||^2 (breakdown threshold)
  __shared__ float coef[LEAF_MAX_W];               // r_{i,t+1}, i <= t
  __shared__ float sc[2];                          // 1/r_tt, r_tt

  const int G = gridDim.x;
  const int g = blockIdx.x;
  const int w = p.w;
  const int RP = p.rows_per_cta;
  const int64_t r0 = (int64_t)g * RP;
  const int64_t rem = p.m - r0;
  const int rows = rem <= 0 ? 0 : (rem < RP ? (int)rem : RP);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  T* P = reinterpret_cast<T*>(p.P);

  // load the slice (coalesced along rows), exact widening to fp32
  for (int j = 0; j < w; ++j)
    for (int i = threadIdx.x; i < RP; i += LEAF_THREADS)
      sp[j * RP + i] = i < rows ? Elem<T>::load(P[r0 + i + (int64_t)j * p.ldp]) : 0.0f;
  __syncthreads();

  const float u_work = 5.9604645e-08f;             // 2^-24, fp32 accumulation
  int bad_first = -1;

  for (int t = 0; t < w; ++t) {
    // ---- 1. local partial sums of this round's vector ----
    int L;
    if (t == 0) L = w + (w > 1 ? 1 : 0);
    else L = (t + 1 < w) ? t + 2 : 1;
    for (int k = warp; k < L; k += LEAF_WARPS) {
      const float* x;
      const float* y;
      if (t == 0) {
        if (k < w) { x = sp + k * RP; y = x; }
        else { x = sp; y = sp + RP; }                           // a_0^T a_1
      } else {
        if (k == 0) { x = sp + t * RP; y = x; }                 // u_t^T u_t
        else if (k == 1) { x = sp + t * RP; y = sp + (t + 1) * RP; }  // u_t^T a_{t+1}
        else { x = sp + (k - 2) * RP; y = sp + (t + 1) * RP; }  // q_i^T a_{t+1}
      }
      float s = 0.0f;
      for (int i = lane; i < rows; i += 32) s = fmaf(x[i], y[i], s);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
      if (lane == 0) p.partials[((int64_t)(t & 1) * (LEAF_MAX_W + 2) + k) * G + g] = s;
    }
    // ---- 2. grid-wide exchange ----
    grid_barrier(p.counter, (unsigned)((t + 1) * G));
    // ---- 3. fixed-order reduction of the G partials (identical in every CTA) ----
    for (int k = warp; k < L; k += LEAF_WARPS) {
      const float* src = p.partials + ((int64_t)(t & 1) * (LEAF_MAX_W + 2) + k) * G;
      float s = 0.0f;
      for (int c = lane; c < G; c += 32) s += __ldcg(src + c);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
      if (lane == 0) tot[k] = s;
    }
    __syncthreads();
    // ---- 4. scalars (thread 0), R entries (CTA 0) ----
    if (threadIdx.x == 0) {
      float uu, ua;
      if (t == 0) {
        for (int k = 0; k < w; ++k) anorm2[k] = tot[k];
        uu = tot[0];
        ua = (w > 1) ? tot[w] : 0.0f;
      } else {
        uu = tot[0];
        ua = (t + 1 < w) ? tot[1] : 0.0f;
      }
      float rtt = sqrtf(uu);
      const float tau = (float)p.m * u_work * sqrtf(anorm2[t]);
      const bool bad = !(rtt > tau) || !isfinite(rtt);
      float inv = 0.0f;
      if (bad) { rtt = 0.0f; if (bad_first < 0) bad_first = t; }
      else inv = 1.0f / rtt;
      sc[0] = inv;
      sc[1] = rtt;
      if (t + 1 < w) {
        for (int i = 0; i < t; ++i) coef[i] = (t == 0) ? 0.0f : tot[2 + i];
        coef[t] = ua * inv;
      }
      if (g == 0) {
        p.R[t + (int64_t)t * p.ldr] = rtt;
        if (t + 1 < w)
          for (int i = 0; i <= t; ++i) p.R[i + (int64_t)(t + 1) * p.ldr] = coef[i];
      }
    }
    __syncthreads();
    // ---- 5. q_t = u_t / r_tt (store rounded), u_{t+1} = a_{t+1} - Q_{<=t} r_{:,t+1} ----
    const float inv = sc[0];
    float* ut = sp + t * RP;
    for (int i = threadIdx.x; i < rows; i += LEAF_THREADS) {
      const float q = ut[i] * inv;
      ut[i] = q;
      P[r0 + i + (int64_t)t * p.ldp] = Elem<T>::store(q);
    }
    __syncthreads();
    if (t + 1 < w) {
      float* a = sp + (t + 1) * RP;
      for (int i = threadIdx.x; i < rows; i += LEAF_THREADS) {
        float u = a[i];
        for (int k = 0; k <= t; ++k) u = fmaf(-sp[k * RP + i], coef[k], u);
        a[i] = u;
      }
    }
    __syncthreads();
  }
  if (g == 0 && threadIdx.x == 0) {
    // zero the strict lower triangle of R11 and report breakdown
    for (int j = 0; j < w; ++j)
      for (int i = j + 1; i < w; ++i) p.R[i + (int64_t)j * p.ldr] = 0.0f;
    if (bad_first >= 0) atomicMin(p.breakdown, (int)(p.col_offset + bad_first));
  }
}

template <typename T>
cudaError_t launch_leaf(const LeafParams& p, int grid, cudaStream_t st) {
  const size_t smem = (size_t)p.w * p.rows_per_cta * sizeof(float);
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
