// tcgen05.mma (cta_group::1, kind::f16, A and B from SW128 shared memory) issue-rate
// micro-benchmark: one CTA per SM, one elected thread issues R rounds of 4 MMAs (K = 64) over
// `stages` 128 x 64 A / N x 64 B k-blocks already in shared memory, commit per k-block, and
// reports cycles per MMA for M = 128 and N in {64, 128, 256}.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I../../paper_conf_hpca_zhaocczlllg22_b200/csrc/kernels
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include "ptx.cuh"
using namespace tk;

__device__ __forceinline__ bool mbar_try(uint64_t *bar, uint32_t parity) {
  uint32_t ok;
  asm volatile("{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
               : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
  return ok != 0;
}
template <int N, int S>
__global__ void __launch_bounds__(128, 1) mma_kernel(int rounds, unsigned long long *cyc, int a_tmem_mode) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t *base = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(sm) + 1023) & ~uintptr_t(1023));
  constexpr uint32_t kA = 288 * 128, kB = N * 128, kStage = kA + kB;
  uint64_t *bar = reinterpret_cast<uint64_t *>(base + S * kStage);
  uint64_t *full = bar + 4, *empty = bar + 4 + S;
  uint32_t *holder = reinterpret_cast<uint32_t *>(bar + 4 + 2 * S);
  for (uint32_t i = threadIdx.x; i < S * kStage / 4; i += 128) reinterpret_cast<uint32_t *>(base)[i] = 0x3c003c00u;
  if (threadIdx.x == 0) {
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], 1);
    mbar_init(&bar[2], 1);
    fence_barrier_init();
    mbar_arrive(&bar[2]);   // phase 0 of bar[2] complete: waits on parity 0 return at once
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    fence_barrier_init();
  }
  if (threadIdx.x < 32) tmem_alloc(holder, 256);
  fence_proxy_async();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *holder;
  constexpr uint32_t idesc = umma_idesc_f16(128, N);
  if (a_tmem_mode >= 3 && a_tmem_mode <= 5 && threadIdx.x >= 32 && threadIdx.x < 64) {   // producer warp: ring handshake only
    int st = 0;
    uint32_t ph = 0;
    for (int i = 0; i < rounds * S; ++i) {
      if (a_tmem_mode == 4) {
        while (!mbar_try(&empty[st], ph ^ 1)) __nanosleep(64);
      } else if (a_tmem_mode == 5) {
        if (threadIdx.x == 32) while (!mbar_try(&empty[st], ph ^ 1)) {}
      } else {
        mbar_wait(&empty[st], ph ^ 1);
      }
      if (elect_one()) mbar_arrive(&full[st]);
      __syncwarp();
      if (++st == S) { st = 0; ph ^= 1; }
    }
  }
  if (a_tmem_mode >= 3 && a_tmem_mode <= 5 && threadIdx.x < 32) {
    unsigned long long t0 = clock64();
    int st = 0;
    uint32_t ph = 0;
    for (int i = 0; i < rounds * S; ++i) {
      mbar_wait(&full[st], ph);
      tc_fence_after();
      if (elect_one()) {
        const uint32_t sa = smem_u32(base + st * kStage), sb = sa + kA;
        const uint64_t da = umma_desc_sw128(sa), db = umma_desc_sw128(sb);
#pragma unroll
        for (int k = 0; k < 4; ++k) umma_f16(tmem, da + 2 * k, db + 2 * k, idesc, (i | k) != 0);
        umma_commit(&empty[st]);
      }
      __syncwarp();
      if (++st == S) { st = 0; ph ^= 1; }
    }
    if (elect_one()) umma_commit(&bar[0]);
    __syncwarp();
    mbar_wait(&bar[0], 0);
    unsigned long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
  } else if (threadIdx.x < 32) {
    unsigned long long t0 = clock64();
    for (int r = 0; r < rounds; ++r) {
      for (int s = 0; s < S; ++s) {
        if (a_tmem_mode == 2) {
          mbar_wait(&bar[2], 0);
          tc_fence_after();
        }
        if (elect_one()) {
          const uint32_t sa = smem_u32(base + s * kStage), sb = sa + kA;
          // mode 6: halo-style A (start s rows in, SBO 1280); mode 7: SBO 2048 (16-pixel pitch), start s rows
          const uint64_t da = a_tmem_mode == 6 ? umma_desc_sw128_sbo(sa + 128 * (r % 3), 1280)
                              : a_tmem_mode == 7 ? umma_desc_sw128_sbo(sa + 128 * (r % 3), 2048)
                              : a_tmem_mode == 8 ? umma_desc_sw128_sbo(sa, 2048)
                                                 : umma_desc_sw128(sa);
          const uint64_t db = umma_desc_sw128(sb);
#pragma unroll
          for (int k = 0; k < 4; ++k) umma_f16(tmem, da + 2 * k, db + 2 * k, idesc, (r | s | k) != 0);
          if (a_tmem_mode == 1) umma_commit(&bar[1]);
        }
        __syncwarp();
      }
    }
    if (elect_one()) umma_commit(&bar[0]);
    __syncwarp();
    mbar_wait(&bar[0], 0);
    unsigned long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
  }
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x < 32) {
    tc_fence_after();
    tmem_dealloc(tmem, 256);
  }
}

template <int N, int S>
void run(int rounds, unsigned long long *d, int mode) {
  const int smem = S * (288 * 128 + N * 128) + 2048 + 1024;
  cudaFuncSetAttribute(mma_kernel<N, S>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  mma_kernel<N, S><<<148, 128, smem>>>(rounds, d, mode);
  cudaDeviceSynchronize();
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  mma_kernel<N, S><<<148, 128, smem>>>(rounds, d, mode);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long h[148];
  cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
  const double mmas = (double)rounds * S * 4;
  double flops = 148.0 * mmas * 2 * 128 * N * 16;
  printf("S=%d mode %d M=128 N=%3d: %.1f cycles/MMA (CTA 0), %.1f TFLOP/s over 148 SMs (%.3f ms)  err=%s\n", S, mode, N, h[0] / mmas,
         flops / (ms * 1e-3) / 1e12, ms, cudaGetErrorString(cudaGetLastError()));
}

int main() {
  unsigned long long *d;
  cudaMalloc(&d, 148 * sizeof(unsigned long long));
  for (int mode : {0, 6, 7, 8}) {
    run<64, 4>(1000, d, mode);
    run<128, 4>(1000, d, mode);
    run<256, 2>(500, d, mode);
  }
  return 0;
}
