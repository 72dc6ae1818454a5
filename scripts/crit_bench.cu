// Micro-benchmark of the leaf's per-column CRITICAL PATH (no bulk work): poll the round's
// 4 exchange words -> broadcast -> scalars -> thread-per-row pass over a 448-row smem slice
// -> warp butterfly -> CTA reduce -> fixed-point red.add.  148 CTAs x 512 threads,
// cooperative launch.  Variants isolate the cost of each step.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o crit_bench crit_bench.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int ROWS = 448, LD = 452, W = 8;
constexpr int SHIFT = 53, VB = 41;

__device__ __forceinline__ unsigned long long ld_rlx(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void red_rlx(unsigned long long* p, unsigned long long v) {
  asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ long long gt() {
  long long v;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(v));
  return v;
}

// variant bits: 1 = float fixed-point conversion (no fp64), 2 = single poller thread for all
// 4 words, 4 = skip the row pass, 8 = skip the butterfly/CTA reduce (thread 0 publishes)
template <int V>
__global__ void __launch_bounds__(512, 1) k_crit(unsigned long long* xw, int rounds, long long* out) {
  __shared__ float sp[W * LD];
  __shared__ float tot[2][4];
  __shared__ float cpart[16][4];
  __shared__ unsigned long long prev[2][4];
  const int G = gridDim.x, g = blockIdx.x, lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < W * LD; i += 512) sp[i] = (i % LD < ROWS) ? 1e-3f * ((i * 7919) % 1000) : 0.f;
  if (threadIdx.x < 8) prev[threadIdx.x >> 2][threadIdx.x & 3] = 0;
  if (threadIdx.x < 8) tot[threadIdx.x >> 2][threadIdx.x & 3] = 1.0f;
  __syncthreads();
  long long t0 = gt();
  float acc = 0.f;
  for (int t = 0; t < rounds; ++t) {
    const int par = t & 1;
    // ---- poll round t's words (published in round t-1) ----
    if (t > 0) {
      if (V & 2) {
        if (threadIdx.x == 0) {
          unsigned long long nw[4];
          bool done = false;
          while (!done) {
#pragma unroll
            for (int k = 0; k < 4; ++k) nw[k] = ld_rlx(xw + (size_t)(par * 4 + k) * 32);
            done = true;
#pragma unroll
            for (int k = 0; k < 4; ++k) done &= (unsigned)((nw[k] - prev[par][k]) >> SHIFT) == (unsigned)G;
          }
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const long long tv = (long long)((nw[k] - prev[par][k]) & ((1ull << SHIFT) - 1)) - (long long)G * (1ll << VB);
            prev[par][k] = nw[k];
            tot[par][k] = (V & 1) ? (float)tv * 0x1p-30f : (float)((double)tv * 0x1p-30);
          }
        }
      } else if (threadIdx.x < 4) {
        const int k = threadIdx.x;
        unsigned long long nw = ld_rlx(xw + (size_t)(par * 4 + k) * 32);
        while ((unsigned)((nw - prev[par][k]) >> SHIFT) != (unsigned)G) nw = ld_rlx(xw + (size_t)(par * 4 + k) * 32);
        const long long tv = (long long)((nw - prev[par][k]) & ((1ull << SHIFT) - 1)) - (long long)G * (1ll << VB);
        prev[par][k] = nw;
        tot[par][k] = (V & 1) ? (float)tv * 0x1p-30f : (float)((double)tv * 0x1p-30);
      }
    }
    __syncthreads();
    // ---- scalars ----
    const float uu = tot[par][0] + 4.0f;
    const float rtt = sqrtf(uu), inv = 1.0f / rtt, ct = tot[par][1] * inv, cq = tot[par][2];
    // ---- row pass ----
    float s0 = 0.f, s1 = 0.f, s2 = 0.f, s3 = 0.f;
    if (!(V & 4)) {
      const int c = t % (W - 4);
      float* ut = sp + c * LD;
      float* an = sp + (c + 1) * LD;
      const float* qp = sp + (c + 2) * LD;
      const float* a2 = sp + (c + 3) * LD;
      const float* a3 = sp + (c + 4 < W ? c + 4 : c) * LD;
      const int r = threadIdx.x;
      if (r < ROWS) {
        const float uv = (V & 32) ? 1.0f : ut[r], av0 = (V & 32) ? 0.5f : an[r], qpv = (V & 32) ? 0.25f : qp[r],
                    a2v = (V & 32) ? 0.1f : a2[r], a3v = (V & 32) ? 0.2f : a3[r];
        const float q = uv * inv;
        if (!(V & 16)) ut[r] = q * 0.999f + 1e-4f;
        float av = fmaf(-qpv, cq * 1e-3f, av0);
        av = fmaf(-q, ct * 1e-3f, av);
        if (!(V & 16)) an[r] = av * 0.999f + 1e-4f;
        s0 = av * av;
        s1 = av * a2v;
        s2 = q * a2v;
        s3 = q * a3v;
      }
    }
    // ---- CTA reduce + publish ----
    if (!(V & 8)) {
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
      __syncthreads();
      if (warp == 15) {
        const int c = lane >> 3, j = lane & 7;
        float s = cpart[j][c] + cpart[j + 8][c];
        s += __shfl_xor_sync(0xffffffffu, s, 4);
        s += __shfl_xor_sync(0xffffffffu, s, 2);
        s += __shfl_xor_sync(0xffffffffu, s, 1);
        if (j == 0) {
          long long v = (V & 1) ? __float2ll_rn(s * 0x1p10f) : __double2ll_rn((double)s * 0x1p10);
          v = v > (1ll << VB) ? (1ll << VB) : (v < -(1ll << VB) ? -(1ll << VB) : v);
          red_rlx(xw + (size_t)(((t + 1) & 1) * 4 + c) * 32, (1ull << SHIFT) + (unsigned long long)(v + (1ll << VB)));
        }
      }
    } else if (threadIdx.x < 4) {
      red_rlx(xw + (size_t)(((t + 1) & 1) * 4 + threadIdx.x) * 32, (1ull << SHIFT) + (1ull << VB));
    }
    acc += s0 + s1 + s2 + s3;
  }
  if (threadIdx.x == 0) out[g] = gt() - t0 + (long long)(acc * 0.f);
}

template <int V>
void run(const char* name, unsigned long long* xw, long long* out, int rounds) {
  void* args[] = {&xw, &rounds, &out};
  for (int rep = 0; rep < 2; ++rep) {
    cudaMemset(xw, 0, 8 * 32 * 8);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    cudaLaunchCooperativeKernel((void*)k_crit<V>, 148, 512, args, 0, 0);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (rep) printf("%-44s %.3f us/round (%s)\n", name, ms * 1e3 / rounds, cudaGetErrorString(cudaGetLastError()));
  }
}

int main() {
  unsigned long long* xw;
  long long* out;
  cudaMalloc(&xw, 8 * 32 * 8);
  cudaMalloc(&out, 160 * 8);
  const int rounds = 20000;
  run<0>("V0 fp64 conv, 4 pollers, rowpass, reduce", xw, out, rounds);
  run<1>("V1 fp32 conv", xw, out, rounds);
  run<2>("V2 one poller for 4 words", xw, out, rounds);
  run<3>("V3 fp32 conv + one poller", xw, out, rounds);
  run<4>("V4 no rowpass", xw, out, rounds);
  run<16>("V16 rowpass loads only", xw, out, rounds);
  run<32>("V32 rowpass stores only", xw, out, rounds);
  run<48>("V48 rowpass arithmetic only", xw, out, rounds);
  run<12>("V12 no rowpass, no reduce (exchange only)", xw, out, rounds);
  run<13>("V13 exchange only, fp32", xw, out, rounds);
  run<15>("V15 exchange only, one poller", xw, out, rounds);
  return 0;
}
