// dtype.cuh -- storage element types of the three precision modes.
#pragma once
#include <cstdint>
#include <cuda_bf16.h>
#include <cuda_fp16.h>

namespace rgsqr {

template <typename T>
struct Elem;

template <>
struct Elem<__half> {
  static constexpr int kBytes = 2;
  static constexpr uint32_t kUmmaFormat = 0;  // F16
  static constexpr bool kTF32 = false;
  __device__ __forceinline__ static float load(__half x) { return __half2float(x); }
  __device__ __forceinline__ static __half store(float x) { return __float2half_rn(x); }
};

template <>
struct Elem<__nv_bfloat16> {
  static constexpr int kBytes = 2;
  static constexpr uint32_t kUmmaFormat = 1;  // BF16
  static constexpr bool kTF32 = false;
  __device__ __forceinline__ static float load(__nv_bfloat16 x) { return __bfloat162float(x); }
  __device__ __forceinline__ static __nv_bfloat16 store(float x) { return __float2bfloat16_rn(x); }
};

template <>
struct Elem<float> {
  static constexpr int kBytes = 4;
  static constexpr uint32_t kUmmaFormat = 2;  // TF32 (reads binary32 smem words)
  static constexpr bool kTF32 = true;
  __device__ __forceinline__ static float load(float x) { return x; }
  __device__ __forceinline__ static float store(float x) { return x; }
};

}  // namespace rgsqr
