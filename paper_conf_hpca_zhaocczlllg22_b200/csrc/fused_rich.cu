// fused_rich.cu — the register-rich class of fused kernels (WMAX = 8: 6 LC + at most 8 BE warps
// per CTA, up to 128 registers per thread instead of 64), compiled in its own translation unit so
// it builds in parallel with tacker_fuse.cu.  tacker_fuse picks it for plans with warp_split <= 8
// (fused.cuh, fused_kernel's WMAX).  Kinds: the bench's BE kernels (Table II
// P:2016-2023 and BASELINE configs 1-4); the others keep the default class only.
#include "kernels/fused.cuh"
#include "runtime.h"

using namespace tk;

namespace tkrt {

using KernelFn = void (*)(FusedParams);

#define TK_FOR_EACH_RICH_BE(X)                                                                   \
  X(TACKER_BE_SGEMM) X(TACKER_BE_STENCIL) X(TACKER_BE_MRIQ_Q) X(TACKER_BE_MRIFHD_FH) X(TACKER_BE_CUTCP) \
  X(TACKER_BE_CP) X(TACKER_BE_LBM) X(TACKER_BE_FFT) X(TACKER_BE_TPACF) X(TACKER_BE_SPMV_JDS)

template <int BN>
static KernelFn rich_fn(int be_kind) {
  switch (be_kind) {
#define C(K) \
  case K: return fused_kernel<BN, K, 8>;
    TK_FOR_EACH_RICH_BE(C)
#undef C
    default: return nullptr;
  }
}

void *pick_fused_rich(int BN, int be_kind) {
  KernelFn f = nullptr;
  if (BN == 64) f = rich_fn<64>(be_kind);
  else if (BN == 128) f = rich_fn<128>(be_kind);
  else if (BN == 256) f = rich_fn<256>(be_kind);
  return reinterpret_cast<void *>(f);
}

}  // namespace tkrt
