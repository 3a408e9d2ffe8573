import sys, os
sys.path.insert(0, os.getcwd())
import torch, paper_conf_ppopp_wintermzss19_b200 as acs
from synth import poisson3d_7pt, aggregation_prolongator
A = poisson3d_7pt(256); P = aggregation_prolongator(256)
dA = acs.DeviceCSR.from_host(A, "cuda"); dP = acs.DeviceCSR.from_host(P, "cuda")
plan = acs.Plan()
for _ in range(2): C = plan.multiply(dA, dP); del C
torch.cuda.synchronize()
