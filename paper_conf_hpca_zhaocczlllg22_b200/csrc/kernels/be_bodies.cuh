// be_bodies.cuh — BE (best-effort, CUDA-core) kernel bodies.
//
// Each body executes ONE original thread block ("virtual block", 128 threads = 4 warps) of a
// Parboil/Rodinia-style kernel given its block id `vb` and the thread id `tid` rebased into
// [0,128) (the "thread_step" of Fig. 5).  Partial-CTA synchronisation uses
// `bar.sync bar_id, 128` (Fig. 9), never __syncthreads().  The same body is
// called by the fused kernel (PTB loop, Fig. 7) and by the original non-persistent kernel,
// so their outputs are bit-identical: all floating-point arithmetic uses explicit
// round-to-nearest intrinsics (no FMA contraction differences between call sites) and a
// per-element order that does not depend on which CTA runs the block.
#pragma once
#include "be_dispatch.cuh"
