"""Table-3-style memory report (Table 3) for the synthetic workloads:
helper memory, chunk pool reserved (exact per-block bound, reading R8) next to the
paper's pool estimate (L556), chunk memory used, used/output (u/o), restarts (always 0:
the deterministic allocator never restarts; the bounded pool defers instead), nnz(C) and the
lowest multiprocessor load
(mpL, L760/L832: min over SMs / max over SMs of the summed block time of each stage-2
kernel that processed blocks, from acspgemm_set_trace / acspgemm_sm_load, reading R36).
Run on a GPU box:
    python tools/table3.py > profiles/r1_table3.md
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_wintermzss19_b200 as acs  # noqa: E402
from synth import aggregation_prolongator, config, poisson3d_7pt  # noqa: E402


def row(name, A, B, dt, pool_mode="exact"):
    vb = np.dtype(dt).itemsize
    dA = acs.DeviceCSR.from_host(A, "cuda", dt)
    dB = dA if B is A else acs.DeviceCSR.from_host(B, "cuda", dt)
    plan = acs.Plan(pool_mode=pool_mode)
    plan.set_trace(True)
    C = plan.multiply(dA, dB)
    torch.cuda.synchronize()
    i = plan.info()
    mpl = []
    for k in ("hash", "rows", "esc", "esc_small"):
        L = plan.sm_load(k)
        if L["blocks"] > 0:
            mpl.append(f"{k} {100 * L['mpl']:.1f} % ({L['blocks']:,})")
    used = i["chunk_elems"] * (4 + vb)
    out = i["nnz_c"] * (4 + vb)
    MB = 1e6
    if pool_mode != "exact":
        name = f"{name} (pool {pool_mode}: {i['ndeferred_blocks']} deferred)"
    line = (f"| {name} | {np.dtype(dt).name} | {i['helper_bytes'] / MB:.1f} | {i['pool_bytes'] / MB:.1f} | "
            f"{i['pool_estimate_bytes'] / MB:.1f} | {used / MB:.1f} | {100 * used / max(i['pool_bytes'], 1):.1f} % | "
            f"{used / max(out, 1):.2f} | 0 | {'; '.join(mpl)} | {i['nnz_c']:,} | {i['nchunks']:,} | {i['nshared']:,} |")
    print(line, flush=True)
    del C, dA, dB
    plan.close()
    torch.cuda.empty_cache()


print("| workload | dtype | helper MB | pool MB (reserved) | pool MB (paper estimate) | used MB | % | u/o | restarts | mpL (kernel, blocks) | nnz(C) | chunks | shared rows |")
print("|---|---|---|---|---|---|---|---|---|---|---|---|---|")
for cfg in ("cfg1", "cfg2", "cfg3", "cfg5"):
    A, B = config(cfg)
    row(cfg, A, B if cfg == "cfg5" else A, np.float64)
A = poisson3d_7pt(256)
row("cfg4a A·P", A, aggregation_prolongator(256), np.float64)
# the bounded pool (acspgemm_options.pool_mode, reading R40): same C, smaller pool
for cfg in ("cfg2",):
    A, B = config(cfg)
    row(cfg, A, A, np.float64, pool_mode="bound")
A = poisson3d_7pt(256)
row("cfg4a A·P", A, aggregation_prolongator(256), np.float64, pool_mode="bound")
