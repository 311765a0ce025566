// Store-path micro-benchmark: write a [M, N] fp16 tensor (M = 100352, N = 256: the b32 layer1 1x1
// conv output, 51 MB) from 148 persistent CTAs of 4 warps, each warp owning 32-row x 64-col boxes,
// by (0) row-strided 16-B STG per thread (thread = row), (1) TMA store of a 32 x 64 SW128 box,
// (2) SMEM transpose + coalesced STG.128 (8 lanes per 128-B row segment), (3) TMA store of a
// 32 x 256 unswizzled box (whole rows).  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lcuda
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int MODE>
__global__ void __launch_bounds__(128, 1) store_kernel(const __grid_constant__ CUtensorMap tm, __half *D, int M, int N) {
  extern __shared__ __align__(1024) uint8_t sm[];
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  uint8_t *stg = sm + warp * 16384;
  int buf = 0;
  const int tiles = (M / 128) * (N / 64);
  for (int t = blockIdx.x; t < tiles; t += gridDim.x) {
    const int mt = t / (N / 64), nt = t % (N / 64);
    const int row = mt * 128 + warp * 32 + lane;
    uint4 val = make_uint4(row, nt, 3, 4);
    if (MODE == 0) {
#pragma unroll
      for (int j = 0; j < 8; ++j) *reinterpret_cast<uint4 *>(D + (size_t)row * N + nt * 64 + 8 * j) = val;
    } else if (MODE == 1) {
      if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      __syncwarp();
      const uint32_t box = smem_u32(stg + buf * 4096) + lane * 128;
#pragma unroll
      for (int j = 0; j < 8; ++j)
        asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(box + ((j ^ (lane & 7)) << 4)), "r"(val.x),
                     "r"(val.y), "r"(val.z), "r"(val.w) : "memory");
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if (lane == 0) {
        asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(&tm),
                     "r"(smem_u32(stg + buf * 4096)), "r"(nt * 64), "r"(mt * 128 + warp * 32) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
      buf ^= 1;
    } else if (MODE == 2) {
      const uint32_t box = smem_u32(stg) + lane * 128;
#pragma unroll
      for (int j = 0; j < 8; ++j)
        asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(box + ((j ^ (lane & 7)) << 4)), "r"(val.x),
                     "r"(val.y), "r"(val.z), "r"(val.w) : "memory");
      __syncwarp();
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int r = 4 * i + lane / 8, c = lane % 8;
        uint4 v;
        asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                     : "r"(smem_u32(stg) + r * 128 + ((c ^ (r & 7)) << 4)));
        *reinterpret_cast<uint4 *>(D + (size_t)(mt * 128 + warp * 32 + r) * N + nt * 64 + 8 * c) = v;
      }
      __syncwarp();
    }
  }
  if (MODE == 1 && lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

int main() {
  const int M = 100352, N = 256;
  __half *D;
  cudaMalloc(&D, (size_t)M * N * 2);
  CUtensorMap tm;
  cuuint64_t dims[2] = {(cuuint64_t)N, (cuuint64_t)M};
  cuuint64_t strides[1] = {(cuuint64_t)N * 2};
  cuuint32_t box[2] = {64, 32}, es[2] = {1, 1};
  CUresult r = cuTensorMapEncodeTiled(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, D, dims, strides, box, es,
                                      CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                                      CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r) printf("encode failed %d\n", r);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  void (*ks[3])(CUtensorMap, __half *, int, int) = {store_kernel<0>, store_kernel<1>, store_kernel<2>};
  const char *names[3] = {"row-strided STG.128 (thread = row)", "TMA store 32x64 SW128 box per warp",
                          "SMEM transpose + coalesced STG.128"};
  for (int m = 0; m < 3; ++m) {
    cudaFuncSetAttribute(ks[m], cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
    for (int it = 0; it < 3; ++it) ks[m]<<<148, 128, 65536>>>(tm, D, M, N);
    cudaEventRecord(e0);
    for (int it = 0; it < 20; ++it) ks[m]<<<148, 128, 65536>>>(tm, D, M, N);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    printf("%-40s %8.2f us  %7.1f GB/s  err=%s\n", names[m], ms * 1e3 / 20, (double)M * N * 2 / (ms / 20 * 1e-3) / 1e9,
           cudaGetErrorString(cudaGetLastError()));
  }
  return 0;
}
