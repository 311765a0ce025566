// be_common.cuh — shared definitions of the BE bodies (see be_bodies.cuh).
#pragma once
#include <cuda_fp16.h>
#include <cstdint>

#include "ptx.cuh"
#include "tacker.h"

namespace tk {
constexpr int kVbThreads = 128;
#ifndef TK_MRIQ_RINT
#define TK_MRIQ_RINT 0   // 1: rintf (FRND) in the mri-q range reduction: measured 0.150 -> 0.189 ms (slow pipe)
#endif
// stencil: planes per thread and resident blocks of the original launch.  Measured (512x512x64,
// standalone): ZC 4 / 8 blocks 31.5 us, ZC 2 / 12 blocks 30 us, ZC 4 / 1 block (74 regs) 37 us;
// fused (ws 24 beside a b1 conv) ZC 4 48 us, ZC 2 55 us -- ZC 4 / 8 blocks kept
#ifndef TK_STENCIL_ZC
#define TK_STENCIL_ZC 4
#endif
#ifndef TK_STENCIL_COARSEN
#define TK_STENCIL_COARSEN 1
#endif
#ifndef TK_STENCIL_MIN_BLOCKS
#define TK_STENCIL_MIN_BLOCKS 8
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
