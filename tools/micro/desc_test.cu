// UMMA shared-memory descriptor semantics for sub-tile starts: A is a 180-row x 64-channel fp16
// "halo" in the SW128 K-major layout (16-byte chunk j of row r at chunk j ^ (r % 8), base 1024-
// aligned), B = identity (64 x 64), so D[m][n] = A[row(m)][n].  The descriptor starts at row r0
// (start = base + 128 r0) with SBO = 1280 B (10 rows between 8-row groups), i.e. row(m) = r0 +
// 10 (m / 8) + m % 8 -- the tap-shifted window of a 16 x 8 output tile over an 18 x 10 halo.
// Checked for several r0 with the base-offset field 0 and = (start >> 7) & 7.
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cstdio>
#include <cstdint>
#include "ptx.cuh"
using namespace tk;

__device__ __forceinline__ uint64_t desc_sw128(uint32_t addr, uint32_t sbo, uint32_t base_off) {
  uint64_t d = 0;
  d |= (uint64_t)((addr & 0x3FFFF) >> 4);
  d |= (uint64_t)(16 >> 4) << 16;
  d |= (uint64_t)((sbo & 0x3FFFF) >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)(base_off & 7) << 49;
  d |= (uint64_t)2 << 61;
  return d;
}

__global__ void __launch_bounds__(128, 1) k(int r0, int bmode, float *out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t *base = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(sm) + 1023) & ~uintptr_t(1023));
  uint8_t *A = base, *B = base + 180 * 128 + 1024 - (180 * 128) % 1024;   // B 1024-aligned after A
  uint64_t *bar = reinterpret_cast<uint64_t *>(B + 64 * 128);
  uint32_t *holder = reinterpret_cast<uint32_t *>(bar + 2);
  for (int i = threadIdx.x; i < 180 * 64; i += 128) {
    const int r = i / 64, c = i % 64;
    const float v = (float)((r * 7 + c * 3) % 17 - 8);
    *reinterpret_cast<__half *>(A + r * 128 + (((c / 8) ^ (r % 8)) << 4) + (c % 8) * 2) = __float2half(v);
  }
  for (int i = threadIdx.x; i < 64 * 64; i += 128) {
    const int n = i / 64, c = i % 64;
    *reinterpret_cast<__half *>(B + n * 128 + (((c / 8) ^ (n % 8)) << 4) + (c % 8) * 2) = __float2half(n == c ? 1.f : 0.f);
  }
  if (threadIdx.x == 0) {
    mbar_init(bar, 1);
    fence_barrier_init();
  }
  if (threadIdx.x < 32) tmem_alloc(holder, 64);
  fence_proxy_async();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *holder;
  if (threadIdx.x < 32) {
    if (elect_one()) {
      const uint32_t start = smem_u32(A) + 128 * r0;
      const uint32_t boff = bmode ? ((start >> 7) & 7) : 0;
      for (int kk = 0; kk < 4; ++kk)
        umma_f16(tmem, desc_sw128(start + 32 * kk, 1280, boff), desc_sw128(smem_u32(B) + 32 * kk, 1024, 0),
                 umma_idesc_f16(128, 64), kk != 0);
      umma_commit(bar);
    }
    __syncwarp();
  }
  mbar_wait(bar, 0);
  tc_fence_after();
  const int w = threadIdx.x / 32;
  uint32_t v[32];
  tmem_ld_32x32b_x32(tmem + ((uint32_t)(w * 32) << 16), v);
  tmem_ld_wait();
  uint32_t v2[32];
  tmem_ld_32x32b_x32(tmem + 32 + ((uint32_t)(w * 32) << 16), v2);
  tmem_ld_wait();
  for (int j = 0; j < 32; ++j) {
    out[threadIdx.x * 64 + j] = __uint_as_float(v[j]);
    out[threadIdx.x * 64 + 32 + j] = __uint_as_float(v2[j]);
  }
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x < 32) {
    tc_fence_after();
    tmem_dealloc(tmem, 64);
  }
}

int main() {
  float *d, h[128 * 64];
  cudaMalloc(&d, sizeof h);
  const int smem = 180 * 128 + 2048 + 64 * 128 + 1024;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  int r0s[] = {0, 1, 2, 3, 7, 8, 10, 11, 12, 20, 21, 22};
  for (int bmode = 0; bmode < 2; ++bmode)
    for (int r0 : r0s) {
      k<<<1, 128, smem>>>(r0, bmode, d);
      cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
      int bad = 0;
      for (int m = 0; m < 128; ++m)
        for (int n = 0; n < 64; ++n) {
          const int r = r0 + 10 * (m / 8) + m % 8;
          const float e = (float)((r * 7 + n * 3) % 17 - 8);
          if (h[m * 64 + n] != e) ++bad;
        }
      printf("base_offset %s r0 %2d: %s (%d of 8192 wrong)  %s\n", bmode ? "=(start>>7)&7" : "= 0         ", r0,
             bad ? "WRONG" : "ok", bad, cudaGetErrorString(cudaGetLastError()));
    }
  return 0;
}
