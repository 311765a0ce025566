// fused_lc.cu — the LC-only (original LC launch) kernels, one instantiation per tile width, LC mode
// and epilogue path (fused.cuh fused_kernel<BN, NONE, 0, MODE, EPI>), in their own translation unit
// (parallel build).  Each carries only its mode's producer / MMA and its epilogue's code: the
// kernel-switch cost of an LC query chain grows with the instruction footprint.
#include "kernels/fused.cuh"
#include "runtime.h"

using namespace tk;

namespace tkrt {

using KernelFn = void (*)(FusedParams);

template <int BN, int EPI>
static KernelFn lc_only_fn(int mode) {
  switch (mode) {
    case kModeGemm: return fused_kernel<BN, TACKER_BE_NONE, 0, kModeGemm, EPI>;
    case kModeIm2col: return fused_kernel<BN, TACKER_BE_NONE, 0, kModeIm2col, EPI>;
    case kModeHalo: return BN <= 128 ? fused_kernel<BN, TACKER_BE_NONE, 0, kModeHalo, EPI> : nullptr;
    case kModeS2c8: return BN == 64 ? fused_kernel<BN, TACKER_BE_NONE, 0, kModeS2c8, EPI> : nullptr;
    case kModeC8: return fused_kernel<BN, TACKER_BE_NONE, 0, kModeC8, EPI>;
    case kModeTiled: return fused_kernel<BN, TACKER_BE_NONE, 0, kModeTiled, EPI>;
    default: return nullptr;
  }
}

void *pick_lc_only_kernel(int BN, int mode, int epi) {
  KernelFn f = nullptr;
  if (epi == 1) {   // the TMA-store epilogue needs 64-column batches
    if (BN == 64) f = lc_only_fn<64, 1>(mode);
    else if (BN == 128) f = lc_only_fn<128, 1>(mode);
    else if (BN == 256) f = lc_only_fn<256, 1>(mode);
  } else {
    if (BN == 64) f = lc_only_fn<64, 2>(mode);
    else if (BN == 128) f = lc_only_fn<128, 2>(mode);
    else if (BN == 256) f = lc_only_fn<256, 2>(mode);
  }
  return reinterpret_cast<void *>(f);
}

}  // namespace tkrt
