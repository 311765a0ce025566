import os, sys
sys.path.insert(0, os.getcwd())
import torch, synth
from paper_conf_hpca_zhaocczlllg22_b200 import services as sv, tacker as tk
convs = [c for c in synth.resnet50_convs(32) if c.name in ("layer1.0.conv3",)]
svc = sv.resnet50_service(32, convs=convs)
k = svc.kernels[0]
for _ in range(3): tk.tacker_launch_original(k.lc, None)
torch.cuda.synchronize(); print("ok")
