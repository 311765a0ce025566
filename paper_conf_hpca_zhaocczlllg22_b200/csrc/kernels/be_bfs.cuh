// be_bfs.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- bfs (Rodinia kernels 1 and 2)
template <> struct BeBody<TACKER_BE_BFS_EXPAND> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_bfs_expand &p) { return (p.V + 127) / 128; }
  static __device__ __forceinline__ void run(const tacker_be_bfs_expand &p, int64_t vb, int tid, uint32_t,
                                             uint8_t *) {
    const int64_t v = vb * 128 + tid;
    if (v >= p.V || !p.mask[v]) return;
    p.mask[v] = 0;
    const int lv = p.level[v] + 1;
    for (int e = p.row_ptr[v]; e < p.row_ptr[v + 1]; ++e) {
      const int u = p.col[e];
      if (!p.visited[u]) {
        p.level[u] = lv;
        p.upd[u] = 1;
      }
    }
  }
};
template <> struct BeBody<TACKER_BE_BFS_COMMIT> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_bfs_commit &p) { return (p.V + 127) / 128; }
  static __device__ __forceinline__ void run(const tacker_be_bfs_commit &p, int64_t vb, int tid, uint32_t,
                                             uint8_t *) {
    const int64_t u = vb * 128 + tid;
    if (u >= p.V || !p.upd[u]) return;
    p.mask[u] = 1;
    p.visited[u] = 1;
    p.upd[u] = 0;
    *p.over = 1;
  }
};

}  // namespace tk
