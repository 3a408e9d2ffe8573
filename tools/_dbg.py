import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import from_coo
def mk(n, step, width):
    r = np.repeat(np.arange(n), 8); c = (np.arange(n)[:, None] + np.arange(8)[None, :]).ravel()
    rng = np.random.default_rng(17)
    A = from_coo(n, n + 8, r, c, rng.uniform(-1, 1, len(r)))
    rb = np.repeat(np.arange(n + 8), width); cb = (step * np.arange(n + 8)[:, None] + np.arange(width)[None, :]).ravel()
    B = from_coo(n + 8, step * (n + 8) + width, rb, cb, rng.uniform(-1, 1, len(rb)))
    return A, B
for step, width in ((5, 30), (1, 30), (2, 30), (3, 30), (4, 30), (5, 40)):
    A, B = mk(3000, step, width)
    dA = acs.DeviceCSR.from_host(A, "cuda", np.float64); dB = acs.DeviceCSR.from_host(B, "cuda", np.float64)
    p = acs.Plan(); C = p.multiply(dA, dB); torch.cuda.synchronize()
    i = p.info(); print(step, width, {k: i[k] for k in ("nblocks", "nhash_blocks", "nrow_blocks", "nchunks", "nshared")}, flush=True)
