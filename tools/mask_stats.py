import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icde_giesekerhvo20_b200 import synth
spec = synth.CONFIGS["landsat"]
Y, dates = synth.generate(spec, "cuda:0")
nan = torch.isnan(Y[:, : 1 << 22]).view(spec.N, -1, 32)
print("missing", nan.float().mean().item(), "warp-date all-missing", nan.all(2).float().mean().item(),
      "all-valid", (~nan).all(2).float().mean().item())
