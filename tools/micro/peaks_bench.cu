// Peak micro-benchmarks for the roofline denominators (SURVEY §8(d) "Peaks"): FP32 FFMA, MUFU
// sin / cos (sin.approx, cos.approx) and rsqrt (rsqrt.approx), fp16 tcgen05.mma (M = 128, N = 256,
// SS operands, 4 k-blocks resident), and an HBM copy.  Each runs on all SMs for ~50-100 ms after a
// warm-up; prints one JSON line (throughputs; the caller records the SM clock).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I../../paper_conf_hpca_zhaocczlllg22_b200/csrc/kernels
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include "ptx.cuh"
using namespace tk;

__global__ void __launch_bounds__(256) ffma_kernel(float *out, int iters, float a, float b) {
  float x[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) x[i] = threadIdx.x * 1e-3f + i;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) x[i] = __fmaf_rn(x[i], a, b);
  }
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < 8; ++i) s += x[i];
  if (s == 12345.f) out[0] = s;
}

__global__ void __launch_bounds__(256) sincos_kernel(float *out, int iters) {
  float x[4], acc = 0.f;
#pragma unroll
  for (int i = 0; i < 4; ++i) x[i] = threadIdx.x * 1e-4f + 0.1f * i;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      float s, c;
      asm volatile("sin.approx.ftz.f32 %0, %1;" : "=f"(s) : "f"(x[i]));
      asm volatile("cos.approx.ftz.f32 %0, %1;" : "=f"(c) : "f"(x[i]));
      x[i] = s + c;
    }
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) acc += x[i];
  if (acc == 12345.f) out[0] = acc;
}

__global__ void __launch_bounds__(256) rsqrt_kernel(float *out, int iters) {
  float x[8], acc = 0.f;
#pragma unroll
  for (int i = 0; i < 8; ++i) x[i] = 1.f + threadIdx.x * 1e-4f + i;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      float r;
      asm volatile("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x[i]));
      x[i] = r + 1.f;
    }
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) acc += x[i];
  if (acc == 12345.f) out[0] = acc;
}

__global__ void __launch_bounds__(128, 1) mma_kernel(int rounds) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t *base = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(sm) + 1023) & ~uintptr_t(1023));
  constexpr uint32_t kA = 128 * 128, kB = 256 * 128, kStage = kA + kB;
  uint64_t *bar = reinterpret_cast<uint64_t *>(base + 4 * kStage);
  uint32_t *holder = reinterpret_cast<uint32_t *>(bar + 2);
  for (uint32_t i = threadIdx.x; i < 4 * kStage / 4; i += 128) reinterpret_cast<uint32_t *>(base)[i] = 0x3c003c00u;
  if (threadIdx.x == 0) {
    mbar_init(bar, 1);
    fence_barrier_init();
  }
  if (threadIdx.x < 32) tmem_alloc(holder, 256);
  fence_proxy_async();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *holder;
  if (threadIdx.x < 32) {
    for (int r = 0; r < rounds; ++r)
      for (int s = 0; s < 4; ++s) {
        if (elect_one()) {
          const uint32_t sa = smem_u32(base + s * kStage);
          const uint64_t da = umma_desc_sw128(sa), db = umma_desc_sw128(sa + kA);
#pragma unroll
          for (int k = 0; k < 4; ++k) umma_f16(tmem, da + 2 * k, db + 2 * k, umma_idesc_f16(128, 256), (r | s | k) != 0);
        }
        __syncwarp();
      }
    if (elect_one()) umma_commit(bar);
    __syncwarp();
    mbar_wait(bar, 0);
  }
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x < 32) {
    tc_fence_after();
    tmem_dealloc(tmem, 256);
  }
}

__global__ void copy_kernel(const float4 *__restrict__ a, float4 *__restrict__ b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) b[i] = a[i];
}

template <typename F>
static float timed(F f, int reps) {
  f();
  cudaDeviceSynchronize();
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float best = 1e30f;
  for (int r = 0; r < reps; ++r) {
    cudaEventRecord(e0);
    f();
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  return best;
}

int main() {
  float *out;
  cudaMalloc(&out, 16);
  const int grid = 148 * 8, block = 256;
  const int it_f = 20000, it_s = 4000, it_r = 8000;
  const float t_f = timed([&] { ffma_kernel<<<grid, block>>>(out, it_f, 1.0000001f, 1e-7f); }, 5);
  const float t_s = timed([&] { sincos_kernel<<<grid, block>>>(out, it_s); }, 5);
  const float t_r = timed([&] { rsqrt_kernel<<<grid, block>>>(out, it_r); }, 5);
  const int smem = 4 * (128 * 128 + 256 * 128) + 2048;
  cudaFuncSetAttribute(mma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int rounds = 4000;
  const float t_m = timed([&] { mma_kernel<<<148, 128, smem>>>(rounds); }, 5);
  const size_t n = (size_t)1 << 28;   // 4 GiB / 16 B... 1 GiB of float4 each way
  float4 *a, *b;
  cudaMalloc(&a, n * 16 / 4);
  cudaMalloc(&b, n * 16 / 4);
  cudaMemset(a, 0, n * 4);
  const float t_c = timed([&] { copy_kernel<<<148 * 16, 512>>>(a, b, n / 4); }, 10);
  const double ffma = (double)grid * block * it_f * 8 * 2 / (t_f * 1e-3) / 1e12;
  const double sincos = (double)grid * block * it_s * 4 * 2 / (t_s * 1e-3) / 1e12;
  const double rsq = (double)grid * block * it_r * 8 / (t_r * 1e-3) / 1e12;
  const double mma = 148.0 * rounds * 16 * 2.0 * 128 * 256 * 16 / (t_m * 1e-3) / 1e12;
  const double hbm = 2.0 * (n / 4) * 16 / (t_c * 1e-3) / 1e9;
  printf("{\"ffma_tflops\": %.2f, \"mufu_sincos_tops\": %.3f, \"mufu_rsqrt_tops\": %.3f, \"f16_tcgen05_tflops\": %.1f, "
         "\"hbm_copy_gbs\": %.1f, \"ms\": {\"ffma\": %.3f, \"sincos\": %.3f, \"rsqrt\": %.3f, \"mma\": %.3f, \"copy\": %.3f}, "
         "\"err\": \"%s\"}\n",
         ffma, sincos, rsq, mma, hbm, t_f, t_s, t_r, t_m, t_c, cudaGetErrorString(cudaGetLastError()));
  return 0;
}
