"""Run one residual-epilogue conv case (name, bn) and print its max error; used under `timeout`."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch, ctypes
import synth
from paper_conf_hpca_zhaocczlllg22_b200 import tacker as tk
name, bn, resid = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
n = int(sys.argv[4]) if len(sys.argv) > 4 else 32
cs = next(c for c in synth.resnet50_convs(n) if c.name == name)
x, w, b = synth.conv_inputs(cs, 99)
res = np.random.default_rng(5).uniform(-1, 1, size=(cs.n, cs.p, cs.q, cs.k)).astype(np.float16)
dx, dw, db, dr = (torch.from_numpy(a).cuda() for a in (x, w, b, res))
out = torch.empty(cs.n, cs.p, cs.q, cs.k, dtype=torch.float16, device="cuda")
lc = tk.lc_conv(dx, dw, out, cs.stride, cs.pad, bias=db, relu=True, residual=dr if resid else None, b_const=True, tile_n=bn)
tk.tacker_launch_original(lc, None)
torch.cuda.synchronize()
print("ok", name, bn, resid, float(out.float().abs().max()), flush=True)
