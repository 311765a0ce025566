"""Launch the kernels the round's ncu captures profile, once each, in this order:
  1. fused ResNet-50 b1 conv (layer3.0.conv2) + mri-q Q chunk (64^3 x 1024 k), warp split 24
  2. fused ResNet-50 b1 conv (layer3.0.conv2) + stencil sweep 512x512x64, warp split 24
  3. ResNet-50 b32 layer3.0.conv2 (LC only, the bench's dominant launch class)
  4. ResNet-50 b32 layer1.0.conv3 (LC only, 1x1, BN 256)
  python tools/ncu_targets.py   (under: ncu --set full -k regex:fused_kernel ...)"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk  # noqa: E402


def main():
    svc1 = sv.resnet50_service(1)
    st, mq = sv.stencil_app(512, 512, 64), sv.mriq_app(64, 2048, 1024)
    tk.tacker_launch_original(None, mq.kernels[0].desc)
    k1 = next(k for k in svc1.kernels if k.name == "layer3.0.conv2")
    f_mq = tk.tacker_fuse(k1.lc, mq.kernels[1].desc, 24)
    f_st = tk.tacker_fuse(k1.lc, st.kernels[0].desc, 24)
    svc32 = sv.resnet50_service(32)
    k32 = {k.name: k for k in svc32.kernels}
    torch.cuda.synchronize()
    f_mq.launch()
    f_st.launch()
    tk.tacker_launch_original(k32["layer3.0.conv2"].lc, None)
    tk.tacker_launch_original(k32["layer1.0.conv3"].lc, None)
    torch.cuda.synchronize()
    print("ok")


if __name__ == "__main__":
    main()
