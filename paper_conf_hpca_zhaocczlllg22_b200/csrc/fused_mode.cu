// fused_mode.cu — fused kernels of the default register class compiled per LC mode (fused.cuh
// fused_kernel<BN, kind, be_max_warps(kind), MODE>) for the BE kinds the bench and the configs
// fuse: like the LC-only kernels (fused_lc.cu), each carries only its LC mode's producer / MMA code
// (the instruction footprint at a kernel switch).  Other kinds / modes: the
// run-time-mode instantiations of tacker_fuse.cu.
#include "kernels/fused.cuh"
#include "runtime.h"

using namespace tk;

namespace tkrt {

using KernelFn = void (*)(FusedParams);

#define TK_FOR_EACH_MODE_BE(X)                                                                    \
  X(TACKER_BE_MRIQ_Q) X(TACKER_BE_MRIFHD_FH) X(TACKER_BE_CP) X(TACKER_BE_LBM) X(TACKER_BE_TPACF)   \
  X(TACKER_BE_STENCIL) X(TACKER_BE_SGEMM) X(TACKER_BE_FFT)

template <int BN, int MODE>
static KernelFn mode_fn(int be_kind) {
  switch (be_kind) {
#define C(K) \
  case K: return fused_kernel<BN, K, be_max_warps(K), MODE>;
    TK_FOR_EACH_MODE_BE(C)
#undef C
    default: return nullptr;
  }
}

void *pick_fused_mode_kernel(int BN, int be_kind, int mode) {
  KernelFn f = nullptr;
  switch (mode) {
    case kModeGemm:
      f = BN == 64 ? mode_fn<64, kModeGemm>(be_kind) : BN == 128 ? mode_fn<128, kModeGemm>(be_kind)
                                                      : BN == 256 ? mode_fn<256, kModeGemm>(be_kind) : nullptr;
      break;
    case kModeIm2col:
      f = BN == 64 ? mode_fn<64, kModeIm2col>(be_kind) : BN == 128 ? mode_fn<128, kModeIm2col>(be_kind)
                                                        : BN == 256 ? mode_fn<256, kModeIm2col>(be_kind) : nullptr;
      break;
    case kModeHalo:
      f = BN == 64 ? mode_fn<64, kModeHalo>(be_kind) : BN == 128 ? mode_fn<128, kModeHalo>(be_kind) : nullptr;
      break;
    default:
      break;
  }
  return reinterpret_cast<void *>(f);
}

}  // namespace tkrt
