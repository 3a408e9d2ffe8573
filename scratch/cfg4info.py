import sys, os, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import poisson3d_7pt, aggregation_prolongator, transpose, config, CSR
A = poisson3d_7pt(256); P = aggregation_prolongator(256)
for strat in ("adaptive", "esc"):
    dA = acs.DeviceCSR.from_host(A, "cuda"); dP = acs.DeviceCSR.from_host(P, "cuda")
    plan = acs.Plan(strategy=strat, stage_times=True)
    for _ in range(3): C = plan.multiply(dA, dP); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(5): C = plan.multiply(dA, dP)
    e1.record(); torch.cuda.synchronize()
    info = plan.info()
    print(strat, e0.elapsed_time(e1) / 5, {k: info[k] for k in ("nblocks", "nrow_blocks", "nhash_blocks", "nshared")}, plan.stage_times(), flush=True)
    plan.close()
