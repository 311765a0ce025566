// be_jds.cuh — see be_bodies.cuh for the conventions shared by all BE bodies.
#pragma once
#include "be_common.cuh"

namespace tk {

// ---------------------------------------------------------------- JDS build (spmv input format)
// Stable counting sort of rows by length, descending, ties by row index:
//   COUNT  per 1024-row block b: c[b][L] = #rows of length L in the block
//   SCAN   per L: c[b][L] -> exclusive prefix over blocks; start[L] = #rows longer than L;
//          jds_ptr[d] = sum_{d' < d} #rows longer than d'
//   PERM   row r of block b with length L goes to start[L] + c[b][L] + (#earlier rows of length
//          L in its block): perm[pos] = r, row_len[pos] = L
//   FILL   element (d, i) = d-th nonzero of row perm[i] at jds_ptr[d] + i
constexpr int kJdsMaxLen = 4095;
constexpr int kJdsRows = 1024;
template <> struct BeBody<TACKER_BE_JDS_COUNT> {
  static constexpr uint32_t kSmem = (kJdsMaxLen + 1) * 4;
  static __host__ __device__ int64_t num_blocks(const tacker_be_jds &p) { return (p.rows + kJdsRows - 1) / kJdsRows; }
  static __device__ __forceinline__ void run(const tacker_be_jds &p, int64_t vb, int tid, uint32_t bar, uint8_t *smem) {
    int32_t *cnt = reinterpret_cast<int32_t *>(smem);
    const int M = p.max_len + 1;
    for (int L = tid; L < M; L += kVbThreads) cnt[L] = 0;
    named_bar_sync(bar, kVbThreads);
    for (int u = 0; u < kJdsRows / kVbThreads; ++u) {
      const int64_t r = vb * kJdsRows + u * kVbThreads + tid;
      if (r < p.rows) {
        const int L = __ldg(p.row_ptr + r + 1) - __ldg(p.row_ptr + r);
        if (L > p.max_len) *p.overflow = 1;
        else atomicAdd(&cnt[L], 1);
      }
    }
    named_bar_sync(bar, kVbThreads);
    for (int L = tid; L < M; L += kVbThreads) p.blk_count[vb * M + L] = cnt[L];
    named_bar_sync(bar, kVbThreads);
  }
};
template <> struct BeBody<TACKER_BE_JDS_SCAN> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_jds &) { return 1; }
  static __device__ __forceinline__ void run(const tacker_be_jds &p, int64_t, int tid, uint32_t bar, uint8_t *) {
    const int M = p.max_len + 1;
    const int64_t nb = (p.rows + kJdsRows - 1) / kJdsRows;
    for (int L = tid; L < M; L += kVbThreads) {
      int32_t s = 0;
      for (int64_t b = 0; b < nb; ++b) {
        const int32_t c = p.blk_count[b * M + L];
        p.blk_count[b * M + L] = s;
        s += c;
      }
      p.start[L] = s;   // total rows of length L
    }
    __threadfence_block();
    named_bar_sync(bar, kVbThreads);
    if (tid == 0) {
      int32_t acc = 0;
      for (int L = M - 1; L >= 0; --L) {   // start[L] = #rows longer than L
        const int32_t t = p.start[L];
        p.start[L] = acc;
        acc += t;
      }
      int32_t ptr = 0;
      for (int d = 0; d < p.max_len; ++d) {
        p.jds_ptr[d] = ptr;
        ptr += p.start[d];
      }
      p.jds_ptr[p.max_len] = ptr;
    }
    named_bar_sync(bar, kVbThreads);
  }
};
template <> struct BeBody<TACKER_BE_JDS_PERM> {
  static constexpr uint32_t kSmem = (kJdsMaxLen + 1) * 4 + kJdsRows * 4;
  static __host__ __device__ int64_t num_blocks(const tacker_be_jds &p) { return (p.rows + kJdsRows - 1) / kJdsRows; }
  static __device__ __forceinline__ void run(const tacker_be_jds &p, int64_t vb, int tid, uint32_t bar, uint8_t *smem) {
    int32_t *cnt = reinterpret_cast<int32_t *>(smem);
    int32_t *lens = cnt + kJdsMaxLen + 1;
    const int M = p.max_len + 1;
    for (int L = tid; L < M; L += kVbThreads) cnt[L] = 0;
    for (int u = 0; u < kJdsRows / kVbThreads; ++u) {
      const int64_t r = vb * kJdsRows + u * kVbThreads + tid;
      lens[u * kVbThreads + tid] =
          r < p.rows ? min(__ldg(p.row_ptr + r + 1) - __ldg(p.row_ptr + r), p.max_len) : -1;
    }
    named_bar_sync(bar, kVbThreads);
    if (tid == 0) {   // rank within the block in row order (stable)
      for (int u = 0; u < kJdsRows; ++u) {
        const int L = lens[u];
        if (L < 0) break;
        const int32_t pos = p.start[L] + p.blk_count[vb * M + L] + cnt[L]++;
        p.perm[pos] = (int32_t)(vb * kJdsRows + u);
        p.row_len[pos] = L;
      }
    }
    named_bar_sync(bar, kVbThreads);
  }
};
template <> struct BeBody<TACKER_BE_JDS_FILL> {
  static constexpr uint32_t kSmem = 0;
  static __host__ __device__ int64_t num_blocks(const tacker_be_jds &p) { return (p.rows + 127) / 128; }
  static __device__ __forceinline__ void run(const tacker_be_jds &p, int64_t vb, int tid, uint32_t, uint8_t *) {
    const int64_t i = vb * 128 + tid;
    if (i >= p.rows) return;
    const int32_t r = p.perm[i], L = p.row_len[i];
    const int32_t base = __ldg(p.row_ptr + r);
    for (int d = 0; d < L; ++d) {
      const int64_t e = (int64_t)p.jds_ptr[d] + i;
      p.jds_col[e] = __ldg(p.col + base + d);
      p.jds_val[e] = __ldg(p.val + base + d);
    }
  }
};

}  // namespace tk
