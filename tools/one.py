"""Two multiplies of one config (for ncu captures).  usage: python tools/one.py CFG [f64|f32] [strategy]"""
import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch, paper_conf_ppopp_wintermzss19_b200 as acs
from synth import config
cfg = sys.argv[1]
dt = np.float32 if len(sys.argv) > 2 and sys.argv[2] == "f32" else np.float64
strategy = sys.argv[3] if len(sys.argv) > 3 else "adaptive"
A, B = config(cfg, dt)
dA = acs.DeviceCSR.from_host(A, "cuda", dt); dB = dA if cfg != "cfg5" else acs.DeviceCSR.from_host(B, "cuda", dt)
plan = acs.Plan(strategy=strategy)
for _ in range(2):
    C = plan.multiply(dA, dB); del C
torch.cuda.synchronize()
