"""Kernels for the PM-sampling overlap evidence (BASELINE: tensor-pipe and FMA-pipe active in the
same intervals of a fused kernel), launched once each in this order:
  1. Table-I analogue: 8192^3 fp16 tcgen05 GEMM || register-only FMA kernel (warp split 24)
  2. the GEMM alone   3. the FMA kernel alone
  4. reverse pair: 4096^3 GEMM || ResNet-50 b32 conv1 im2col (warp split 24)
  python tools/pm_targets.py   (under: ncu --section PmSampling -k regex:"fused_kernel|be_original")"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk  # noqa: E402


def main():
    A, B = synth.lc_gemm_inputs(8192, 8192, 8192, seed=0)
    dA, dB = torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda()
    D = torch.empty(8192, 8192, device="cuda")
    lc = tk.lc_gemm(dA, dB, D)
    out = torch.empty(tk.tacker_device_sm_count() * 24 * 32, device="cuda")
    kc = tk.be_fma_burn(out, 60000)
    f = tk.tacker_fuse(lc, kc, 24)
    train = sv.gemm_train_app(4096, 4096, 4096, n=1)
    c1 = sv.resnet50_service(32, convs=synth.resnet50_convs(32)[:1], conv1_im2col=True)
    fr = tk.tacker_fuse(train.kernels[0].desc, c1.kernels[0].cd, 24)
    torch.cuda.synchronize()
    f.launch()
    tk.tacker_launch_original(lc, None)
    tk.tacker_launch_original(None, kc)
    fr.launch()
    torch.cuda.synchronize()
    print("ok")


if __name__ == "__main__":
    main()
