import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
from oracle import be as obe
from oracle.metrics import max_rel_err
from paper_conf_hpca_zhaocczlllg22_b200 import tacker as tk
mode = sys.argv[1]
nx, ny, nz = (int(x) for x in sys.argv[2:5])
A = synth.stencil_inputs(nx, ny, nz, 1)
dA = torch.from_numpy(A).cuda(); dN = torch.zeros_like(dA)
d = tk.be_stencil(dA, dN)
print("blocks", tk.tacker_be_num_blocks(d), flush=True)
if mode == "orig":
    tk.tacker_launch_original(None, d)
else:
    a = torch.zeros(128, 64, dtype=torch.float16, device="cuda"); D = torch.zeros(128, 128, device="cuda")
    f = tk.tacker_fuse(tk.lc_gemm(a, a[:, :64].contiguous() if False else torch.zeros(128, 64, dtype=torch.float16, device="cuda"), D), d, int(sys.argv[5]))
    print(f.info().smem_bytes, flush=True)
    f.launch()
torch.cuda.synchronize()
ref, S = obe.stencil(A, np.float32(1/6), np.float32(1/36))
print(mode, "err", max_rel_err(dN.cpu().numpy(), ref, S), flush=True)
