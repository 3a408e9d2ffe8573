import sys, os
sys.path.insert(0, os.getcwd())
import torch, paper_conf_ppopp_wintermzss19_b200 as acs
from synth import config
cfg = sys.argv[1]
A, B = config(cfg)
dA = acs.DeviceCSR.from_host(A, "cuda"); dB = dA if cfg != "cfg5" else acs.DeviceCSR.from_host(B, "cuda")
plan = acs.Plan()
for _ in range(2):
    C = plan.multiply(dA, dB); del C
torch.cuda.synchronize()
