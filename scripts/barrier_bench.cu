// Micro-benchmark of grid-wide exchange variants for the leaf CGS rounds (148 CTAs x 256 threads).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o barrier_bench barrier_bench.cu
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned ld_acq(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_rel(unsigned* p, unsigned v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// (a) one counter, atomicAdd + spin by thread 0
__global__ void k_counter(unsigned* cnt, int rounds, int sleep_ns) {
  for (int t = 0; t < rounds; ++t) {
    __syncthreads();
    if (threadIdx.x == 0) {
      __threadfence();
      atomicAdd(cnt, 1u);
      unsigned target = (t + 1) * gridDim.x;
      while (ld_acq(cnt) < target) {
        if (sleep_ns) __nanosleep(sleep_ns);
      }
    }
    __syncthreads();
  }
}

// (b) per-CTA flags, warp 0 polls all flags in parallel
__global__ void k_flags(unsigned* flags, int rounds) {
  const int G = gridDim.x;
  for (int t = 0; t < rounds; ++t) {
    __syncthreads();
    if (threadIdx.x == 0) st_rel(flags + blockIdx.x * 32, t + 1);   // own 128-B line
    if (threadIdx.x < 32) {
      bool done;
      do {
        done = true;
        for (int c = threadIdx.x; c < G; c += 32) done &= ld_acq(flags + c * 32) >= (unsigned)(t + 1);
      } while (!__all_sync(0xffffffffu, done));
    }
    __syncthreads();
  }
}

// (c) red.release add (no return) + spin
__global__ void k_red(unsigned* cnt, int rounds) {
  for (int t = 0; t < rounds; ++t) {
    __syncthreads();
    if (threadIdx.x == 0) {
      asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(cnt) : "memory");
      unsigned target = (t + 1) * gridDim.x;
      while (ld_acq(cnt) < target) {
      }
    }
    __syncthreads();
  }
}

// (d) data exchange: each CTA writes L partials then counter barrier, then all read G*L (batched)
__global__ void k_exchange(unsigned* cnt, float* part, int rounds, int L) {
  const int G = gridDim.x;
  __shared__ float tot[80];
  for (int t = 0; t < rounds; ++t) {
    float* buf = part + (t & 1) * 80 * 160;
    if (threadIdx.x < L) buf[threadIdx.x * G + blockIdx.x] = (float)(t + threadIdx.x);
    __syncthreads();
    if (threadIdx.x == 0) {
      __threadfence();
      atomicAdd(cnt, 1u);
      unsigned target = (t + 1) * gridDim.x;
      while (ld_acq(cnt) < target) {
      }
    }
    __syncthreads();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    float v[9][5];
#pragma unroll
    for (int a = 0; a < 9; ++a)
#pragma unroll
      for (int q = 0; q < 5; ++q) {
        int k = warp + a * 8, c = lane + 32 * q;
        v[a][q] = (k < L && c < G) ? __ldcg(buf + k * G + c) : 0.f;
      }
#pragma unroll
    for (int a = 0; a < 9; ++a) {
      float s = v[a][0] + v[a][1] + v[a][2] + v[a][3] + v[a][4];
      for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
      if (lane == 0 && warp + a * 8 < L) tot[warp + a * 8] = s;
    }
    __syncthreads();
  }
  if (threadIdx.x == 0 && blockIdx.x == 0) part[0] = tot[0];
}

int main() {
  unsigned* cnt;
  float* part;
  cudaMalloc(&cnt, 160 * 32 * 4);
  cudaMalloc(&part, 2 * 80 * 160 * 4);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int rounds = 2000;
  int grids[] = {148, 74, 32, 16};
  for (int G : grids) {
    for (int variant = 0; variant < 6; ++variant) {
      cudaMemset(cnt, 0, 160 * 32 * 4);
      void* args0[] = {&cnt, (void*)&rounds, nullptr};
      int sl = variant == 1 ? 32 : (variant == 2 ? 200 : 0);
      int L = variant == 5 ? 34 : 0;
      cudaEventRecord(a);
      if (variant <= 2) {
        void* args[] = {&cnt, (void*)&rounds, &sl};
        cudaLaunchCooperativeKernel((void*)k_counter, G, 256, args, 0, 0);
      } else if (variant == 3) {
        void* args[] = {&cnt, (void*)&rounds};
        cudaLaunchCooperativeKernel((void*)k_flags, G, 256, args, 0, 0);
      } else if (variant == 4) {
        void* args[] = {&cnt, (void*)&rounds};
        cudaLaunchCooperativeKernel((void*)k_red, G, 256, args, 0, 0);
      } else {
        void* args[] = {&cnt, &part, (void*)&rounds, &L};
        cudaLaunchCooperativeKernel((void*)k_exchange, G, 256, args, 0, 0);
      }
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      const char* names[] = {"counter", "counter+sleep32", "counter+sleep200", "flags", "red.release", "exchange L=34"};
      printf("G=%3d %-18s %.3f us/round (%s)\n", G, names[variant], ms * 1e3 / rounds,
             cudaGetErrorString(cudaGetLastError()));
      (void)args0;
    }
  }
  return 0;
}
