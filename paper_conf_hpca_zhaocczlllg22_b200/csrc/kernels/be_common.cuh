// be_common.cuh — shared definitions of the BE bodies (see be_bodies.cuh).
#pragma once
#include <cuda_fp16.h>
#include <cstdint>

#include "ptx.cuh"
#include "tacker.h"

namespace tk {
constexpr int kVbThreads = 128;
#ifndef TK_STENCIL_ZC
#define TK_STENCIL_ZC 4
#endif
#ifndef TK_STENCIL_HOIST
#define TK_STENCIL_HOIST 0
#endif
#ifndef TK_MRIQ_COARSEN
#define TK_MRIQ_COARSEN 4
#endif
#ifndef TK_FFT_MAXN
#define TK_FFT_MAXN 1024
#endif
#ifndef TK_FFT_ODD_FIRST
#define TK_FFT_ODD_FIRST 1   // fft: the radix-2^f pass first (n = 256: 98.6 -> 90.7 us; equal at 1024)
#endif
#ifndef TK_FFT_PER_BLOCK
#define TK_FFT_PER_BLOCK 2   // fft: transforms per original block (n = 256: 80 -> 72 us; equal at 1024)
#endif
#ifndef TK_FFT_MIN_BLOCKS
#define TK_FFT_MIN_BLOCKS 8  // fft original grid: 64 registers, no spills with two transforms per block
#endif
#ifndef TK_MRIQ_REDUCE
// mri-q / mri-fhd: exact range reduction of the phase in turns, t - rint(t), before the MUFU
// sin/cos of 2 pi t: |2 pi t| <= pi, where sin.approx / cos.approx hold their
// 2^-20.9 absolute error bound (the bench's k in [-32, 32) puts |t| up to 48 turns).  Two FADDs
// per term on the FMA pipe beside the MUFU-bound sin/cos.
#define TK_MRIQ_REDUCE 1
#endif

template <int KIND> struct BeBody;

}  // namespace tk
