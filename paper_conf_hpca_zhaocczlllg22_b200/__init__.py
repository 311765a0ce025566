"""B200-native Tacker: Tensor-CUDA core fused kernels (tcgen05 LC GEMM/conv + CUDA-core BE
bodies in one persistent CTA), a two-stage duration predictor and a QoS-aware kernel manager,
behind the C ABI in include/tacker.h (libtacker.so).  See DESIGN.md.

Import `paper_conf_hpca_zhaocczlllg22_b200.tacker` for the binding; it fails loudly if the
CUDA library is not built (there is no CPU fallback).
"""
__all__ = ["tacker", "build"]
