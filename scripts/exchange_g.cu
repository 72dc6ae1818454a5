// Micro-benchmark of the leaf's fixed-point all-reduce (one round = every CTA contributes L values,
// every CTA needs the L totals), no compute.  148 CTAs x 512 threads, cooperative launch.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o exchange_bench exchange_bench.cu
//
//   A  per-word polling, C word copies (CTA g adds into copy g % C), L*C polling threads
//   B  flag word: data reds relaxed, then bar.sync + one red.release on a counter word;
//      thread 0 polls the counter (acquire), then L threads read the data words once
//   E  cluster pre-reduction (cluster of CL CTAs, DSMEM), leader adds, per-word polling by every CTA
#include <cooperative_groups.h>
#include <cstdio>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;

constexpr int MAXL = 66;
constexpr int MAXC = 8;
constexpr int SHIFT = 53;

__device__ __forceinline__ unsigned long long ld_rlx(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ld_acq64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void red_rlx(unsigned long long* p, unsigned long long v) {
  asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void red_rel(unsigned long long* p, unsigned long long v) {
  asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// A: per-word polling
__global__ void __launch_bounds__(512, 1) k_poll(unsigned long long* xw, int rounds, int L, int C, int sleep_ns,
                                                long long* out, int S) {
  __shared__ unsigned long long prev[2 * MAXL * MAXC];
  __shared__ long long tot[MAXL];
  for (int i = threadIdx.x; i < 2 * MAXL * MAXC; i += blockDim.x) prev[i] = 0;
  const int G = gridDim.x, g = blockIdx.x;
  __syncthreads();
  long long acc = 0;
  for (int t = 0; t < rounds; ++t) {
    if (threadIdx.x < L) {
      const int k = threadIdx.x;
      red_rlx(xw + (size_t)(((t & 1) * MAXL + k) * MAXC + g % C) * S, (1ull << SHIFT) + (unsigned long long)(g + k + t));
    }
    const int k = threadIdx.x / C, h = threadIdx.x % C;
    long long v = 0;
    if (k < L) {
      const int wi = ((t & 1) * MAXL + k) * MAXC + h;
      const unsigned cnt = G / C + (h < G % C ? 1 : 0);
      unsigned long long now = ld_rlx(xw + (size_t)wi * S), d = now - prev[wi];
      long long spins = 0;
      while ((unsigned)(d >> SHIFT) != cnt && ++spins < (1ll << 24)) {
        if (sleep_ns) __nanosleep(sleep_ns);
        now = ld_rlx(xw + (size_t)wi * S);
        d = now - prev[wi];
      }
      prev[wi] = now;
      v = (long long)(d & ((1ull << SHIFT) - 1));
    }
    for (int o = 1; o < C; o <<= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (k < L && h == 0) tot[k] = v;
    __syncthreads();
    acc += tot[t % L];
  }
  if (threadIdx.x == 0) out[g] = acc;
}

// B: data words + release counter
__global__ void __launch_bounds__(512, 1) k_flag(unsigned long long* xw, unsigned long long* ctr, int rounds, int L,
                                                long long* out) {
  __shared__ long long tot[MAXL];
  __shared__ unsigned long long prevd[2 * MAXL];
  const int G = gridDim.x, g = blockIdx.x;
  for (int i = threadIdx.x; i < 2 * MAXL; i += blockDim.x) prevd[i] = 0;
  __syncthreads();
  long long acc = 0;
  for (int t = 0; t < rounds; ++t) {
    if (threadIdx.x < L) red_rlx(xw + (t & 1) * MAXL + threadIdx.x, (unsigned long long)(g + threadIdx.x + t));
    __syncthreads();
    if (threadIdx.x == 0) {
      red_rel(ctr, 1ull);
      const unsigned long long target = (unsigned long long)(t + 1) * G;
      long long spins = 0;
      while (ld_acq64(ctr) < target && ++spins < (1ll << 24)) {
      }
    }
    __syncthreads();
    if (threadIdx.x < L) {
      const int wi = (t & 1) * MAXL + threadIdx.x;
      const unsigned long long now = ld_rlx(xw + wi);
      tot[threadIdx.x] = (long long)(now - prevd[wi]);
      prevd[wi] = now;
    }
    __syncthreads();
    acc += tot[t % L];
  }
  if (threadIdx.x == 0) out[g] = acc;
}

// E: cluster pre-reduction over DSMEM, leader CTA adds one partial per value
template <int CL>
__global__ void __cluster_dims__(CL, 1, 1) __launch_bounds__(512, 1)
    k_cluster(unsigned long long* xw, int rounds, int L, long long* out) {
  __shared__ unsigned long long prev[2 * MAXL];
  __shared__ long long tot[MAXL];
  __shared__ long long mine[2][MAXL];
  cg::cluster_group cl = cg::this_cluster();
  const int G = gridDim.x, g = blockIdx.x;
  const int NC = G / CL;
  for (int i = threadIdx.x; i < 2 * MAXL; i += blockDim.x) prev[i] = 0;
  __syncthreads();
  long long acc = 0;
  for (int t = 0; t < rounds; ++t) {
    if (threadIdx.x < L) mine[t & 1][threadIdx.x] = g + threadIdx.x + t;
    cl.sync();
    if (cl.block_rank() == 0 && threadIdx.x < L) {
      long long s = 0;
      for (int r = 0; r < CL; ++r) s += cl.map_shared_rank(&mine[t & 1][0], r)[threadIdx.x];
      red_rlx(xw + (t & 1) * MAXL + threadIdx.x, (1ull << SHIFT) + (unsigned long long)s);
    }
    if (threadIdx.x < L) {
      const int wi = (t & 1) * MAXL + threadIdx.x;
      unsigned long long now = ld_rlx(xw + wi), d = now - prev[wi];
      long long spins = 0;
      while ((unsigned)(d >> SHIFT) != (unsigned)NC && ++spins < (1ll << 24)) {
        now = ld_rlx(xw + wi);
        d = now - prev[wi];
      }
      prev[wi] = now;
      tot[threadIdx.x] = (long long)(d & ((1ull << SHIFT) - 1));
    }
    __syncthreads();
    acc += tot[t % L];
  }
  cl.sync();
  if (threadIdx.x == 0) out[g] = acc;
}

// A2: per-word polling, spread words (stride S words), D loads in flight per polling thread
template <int D>
__global__ void __launch_bounds__(512, 1) k_poll_pipe(unsigned long long* xw, int rounds, int L, long long* out, int S) {
  __shared__ unsigned long long prev[2 * MAXL];
  __shared__ long long tot[MAXL];
  for (int i = threadIdx.x; i < 2 * MAXL; i += blockDim.x) prev[i] = 0;
  const int G = gridDim.x, g = blockIdx.x;
  __syncthreads();
  long long acc = 0;
  for (int t = 0; t < rounds; ++t) {
    if (threadIdx.x < L)
      red_rlx(xw + (size_t)((t & 1) * MAXL + threadIdx.x) * S, (1ull << SHIFT) + (unsigned long long)(g + threadIdx.x + t));
    if (threadIdx.x < L) {
      const int wi = (t & 1) * MAXL + threadIdx.x;
      const unsigned long long* wp = xw + (size_t)wi * S;
      const unsigned long long pv = prev[wi];
      unsigned long long v[D];
#pragma unroll
      for (int j = 0; j < D; ++j) v[j] = ld_rlx(wp);
      unsigned long long now = 0;
      bool done = false;
      long long spins = 0;
      while (!done && ++spins < (1ll << 22)) {
#pragma unroll
        for (int j = 0; j < D; ++j) {
          if (!done) {
            if ((unsigned)((v[j] - pv) >> SHIFT) == (unsigned)G) { done = true; now = v[j]; }
            else v[j] = ld_rlx(wp);
          }
        }
      }
      prev[wi] = now;
      tot[threadIdx.x] = (long long)((now - pv) & ((1ull << SHIFT) - 1));
    }
    __syncthreads();
    acc += tot[t % L];
  }
  if (threadIdx.x == 0) out[g] = acc;
}

template <typename K>
int max_clusters(K kern, int cl) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(148);
  cfg.blockDim = dim3(512);
  cudaLaunchAttribute at;
  at.id = cudaLaunchAttributeClusterDimension;
  at.val.clusterDim.x = cl;
  at.val.clusterDim.y = 1;
  at.val.clusterDim.z = 1;
  cfg.attrs = &at;
  cfg.numAttrs = 1;
  int n = 0;
  cudaOccupancyMaxActiveClusters(&n, (void*)kern, &cfg);
  printf("max active clusters of %d: %d\n", cl, n);
  return n;
}


int main() {
  unsigned long long *xw, *ctr;
  long long* out;
  cudaMalloc(&xw, 2 * MAXL * MAXC * 8 * 128);
  cudaMalloc(&ctr, 8);
  cudaMalloc(&out, 160 * 8);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  int rounds = 4000;
  auto run = [&](const char* name, auto launch) {
    cudaMemset(xw, 0, 2 * MAXL * MAXC * 8 * 128);
    cudaMemset(ctr, 0, 8);
    launch();
    cudaMemset(xw, 0, 2 * MAXL * MAXC * 8 * 128);
    cudaMemset(ctr, 0, 8);
    cudaEventRecord(a);
    launch();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    printf("%-40s %.3f us/round (%s)\n", name, ms * 1e3 / rounds, cudaGetErrorString(cudaGetLastError()));
  };
  for (int G : {148, 128, 96, 74, 48, 37, 16, 8, 2}) {
    int L = 4, S = 32;
    char nm[96];
    snprintf(nm, sizeof nm, "G=%d A2 pipe4 L=%d", G, L);
    run(nm, [&] { void* args[] = {&xw, &rounds, &L, &out, &S};
      cudaLaunchCooperativeKernel((void*)k_poll_pipe<4>, G, 512, args, 0, 0); });
    int C = 1, sl = 0;
    snprintf(nm, sizeof nm, "G=%d A poll L=%d", G, L);
    run(nm, [&] { void* args[] = {&xw, &rounds, &L, &C, &sl, &out, &S};
      cudaLaunchCooperativeKernel((void*)k_poll, G, 512, args, 0, 0); });
  }
  return 0;
}
