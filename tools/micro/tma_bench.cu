// TMA load throughput from L2: 148 CTAs (1 per SM), one elected thread streams 16 KB boxes
// (128 rows x 128 B, SW128) into an S-stage ring, a consumer warp only waits and releases.
// Modes: 0 = 2-D tiled box of a [rows, 64] fp16 matrix; 1 = im2col 4-D box (128 pixels x 64 ch,
// 3x3 tap offsets cycling) of an NHWC tensor; 2 = 4-D tiled box {64, 10, 16, 1} (a 20 KB conv halo).
// The source (32 MB) stays L2-resident.  Reports B/clk/SM and TB/s.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include "ptx.cuh"
using namespace tk;

template <int MODE>
__global__ void __launch_bounds__(64, 1) k(const __grid_constant__ CUtensorMap tm, int iters, int S, unsigned long long *cyc) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t *base = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(sm) + 1023) & ~uintptr_t(1023));
  constexpr uint32_t kBox = MODE == 2 ? 160 * 128 : 128 * 128;
  constexpr uint32_t kSlot = (kBox + 1023) & ~1023u;
  uint64_t *full = reinterpret_cast<uint64_t *>(base + 8 * kSlot), *empty = full + 8;
  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    fence_barrier_init();
  }
  __syncthreads();
  const unsigned long long t0 = clock64();
  if (threadIdx.x < 32) {
    int st = 0;
    uint32_t ph = 0;
    for (int i = 0; i < iters; ++i) {
      mbar_wait(&empty[st], ph ^ 1);
      if (elect_one()) {
        mbar_arrive_expect_tx(&full[st], kBox);
        const int j = (blockIdx.x * 37 + i) % 1000;
        if (MODE == 0) tma_load_2d(&tm, &full[st], base + st * kSlot, 0, j * 128);
        else if (MODE == 1) tma_load_im2col_4d(&tm, &full[st], base + st * kSlot, 0, (j % 7) * 8 - 1, (j / 7) % 56 - 1, j % 8, i % 3, (i / 3) % 3);
        else tma_load_4d(&tm, &full[st], base + st * kSlot, 0, (j % 7) * 8 - 1, (j / 7) % 56 - 1, j % 8);
      }
      __syncwarp();
      if (++st == S) { st = 0; ph ^= 1; }
    }
  } else {
    int st = 0;
    uint32_t ph = 0;
    for (int i = 0; i < iters; ++i) {
      mbar_wait(&full[st], ph);
      if (elect_one()) mbar_arrive(&empty[st]);
      __syncwarp();
      if (++st == S) { st = 0; ph ^= 1; }
    }
    if (threadIdx.x == 32) cyc[blockIdx.x] = clock64() - t0;
  }
}

using PFN_im2col = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                const cuuint64_t *, const int *, const int *, cuuint32_t, cuuint32_t,
                                const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion,
                                CUtensorMapFloatOOBfill);

int main() {
  const int n = 8, h = 56, w = 56, c = 64;     // 3.2 MB NHWC (one b8 layer1 activation) ... x 10 below
  void *x;
  const size_t bytes = 32ull << 20;
  cudaMalloc(&x, bytes);
  cudaMemset(x, 0, bytes);
  unsigned long long *d;
  cudaMalloc(&d, 148 * sizeof(unsigned long long));
  CUtensorMap t2, ti, t4;
  cuuint64_t d2[2] = {64, bytes / 128}, s2[1] = {128};
  cuuint32_t b2[2] = {64, 128}, e2[2] = {1, 1};
  cuTensorMapEncodeTiled(&t2, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, x, d2, s2, b2, e2, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  cuuint64_t d4[4] = {(cuuint64_t)c, (cuuint64_t)w, (cuuint64_t)h, (cuuint64_t)n};
  cuuint64_t s4[3] = {(cuuint64_t)c * 2, (cuuint64_t)c * w * 2, (cuuint64_t)c * w * h * 2};
  int lo[2] = {-1, -1}, hi[2] = {-1, -1};
  cuuint32_t e4[4] = {1, 1, 1, 1};
  void *fp = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &fp, cudaEnableDefault, &q);
  reinterpret_cast<PFN_im2col>(fp)(&ti, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4, x, d4, s4, lo, hi, 64, 128, e4,
                                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  cuuint32_t b4[4] = {64, 10, 16, 1};
  cuTensorMapEncodeTiled(&t4, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4, x, d4, s4, b4, e4, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  const int smem = 8 * 21504 + 2048;
  const char *names[3] = {"2-D tiled 128 x 128 B", "im2col 128 px x 128 B (3x3 taps)", "4-D tiled halo 16x10 px x 128 B"};
  for (int mode = 0; mode < 3; ++mode)
    for (int S : {2, 4, 8}) {
      auto fn = mode == 0 ? k<0> : mode == 1 ? k<1> : k<2>;
      const CUtensorMap &tm = mode == 0 ? t2 : mode == 1 ? ti : t4;
      cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      const int iters = 4000;
      fn<<<148, 64, smem>>>(tm, iters, S, d);
      cudaEvent_t e0, e1;
      cudaEventCreate(&e0);
      cudaEventCreate(&e1);
      cudaEventRecord(e0);
      fn<<<148, 64, smem>>>(tm, iters, S, d);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      unsigned long long hcyc[148];
      cudaMemcpy(hcyc, d, sizeof hcyc, cudaMemcpyDeviceToHost);
      const double box = mode == 2 ? 160 * 128 : 128 * 128;
      printf("%-34s S=%d: %6.1f B/clk/SM (CTA 0), %6.2f TB/s chip  %s\n", names[mode], S, box * iters / hcyc[0],
             148.0 * box * iters / (ms * 1e-3) / 1e12, cudaGetErrorString(cudaGetLastError()));
    }
  return 0;
}
