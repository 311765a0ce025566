"""Launch the kernels the round's ncu captures profile, once each, in this order:
  1. fused ResNet-50 b1 conv (layer3.0.conv2) + mri-q Q chunk (64^3 x 1024 k), warp split 24
  2. fused ResNet-50 b1 conv (layer3.0.conv2) + stencil sweep 512x512x64, warp split 24
  3. ResNet-50 b32 layer3.0.conv2 (LC only, the bench's dominant launch class; im2col-mode TMA)
  4. ResNet-50 b32 layer1.0.conv3 (LC only, 1x1, BN 256)
  with --next3 also (NEXT-3 / NEXT-2, each fused with the b1 conv at warp split 24 unless noted):
  5. fused conv + mri-fhd FH chunk   6. fused conv + cp slice   7. fused conv + fft (ws 24)
  8. fused conv + tpacf DR (ws 16)   9. reverse: 4096^3 fp16 GEMM (tcgen05) + b32 conv1 im2col (ws 24)
  python tools/ncu_targets.py [--next3]   (under: ncu --set full -k regex:fused_kernel ...)"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk  # noqa: E402


def main():
    next3 = "--next3" in sys.argv
    svc1 = sv.resnet50_service(1)
    st, mq = sv.stencil_app(512, 512, 64), sv.mriq_app(64, 2048, 1024)
    tk.tacker_launch_original(None, mq.kernels[0].desc)
    k1 = next(k for k in svc1.kernels if k.name == "layer3.0.conv2")
    f_mq = tk.tacker_fuse(k1.lc, mq.kernels[1].desc, 24)
    f_st = tk.tacker_fuse(k1.lc, st.kernels[0].desc, 24)
    svc32 = sv.resnet50_service(32)
    k32 = {k.name: k for k in svc32.kernels}
    extra = []
    if next3:
        fh, cp, ff, tp = sv.mrifhd_app(), sv.cp_app(), sv.fft_app(), sv.tpacf_app()
        tk.tacker_launch_original(None, fh.kernels[0].desc)
        train = sv.gemm_train_app(4096, 4096, 4096, n=1)
        c1 = sv.resnet50_service(32, convs=synth.resnet50_convs(32)[:1], conv1_im2col=True)
        extra = [tk.tacker_fuse(k1.lc, fh.kernels[1].desc, 24), tk.tacker_fuse(k1.lc, cp.kernels[0].desc, 24),
                 tk.tacker_fuse(k1.lc, ff.kernels[0].desc, 24), tk.tacker_fuse(k1.lc, tp.kernels[1].desc, 16),
                 tk.tacker_fuse(train.kernels[0].desc, c1.kernels[0].cd, 24)]
        keep = (fh, cp, ff, tp, train, c1)  # noqa: F841
    torch.cuda.synchronize()
    f_mq.launch()
    f_st.launch()
    tk.tacker_launch_original(k32["layer3.0.conv2"].lc, None)
    tk.tacker_launch_original(k32["layer1.0.conv3"].lc, None)
    for f in extra:
        f.launch()
    torch.cuda.synchronize()
    print("ok")


if __name__ == "__main__":
    main()
