"""E5 analog (webbase-1M at 0/3/5/10/21/42/63 restarts): the cost of
running a multiply within a shrinking chunk-pool budget (acspgemm_multiply_budget:
pieces of whole canonical segments, a refused piece retried on fewer segments).  The
result is bit-identical for every budget; the table reports time, pieces, restarts.
Run on a GPU box:  python tools/restart_sweep.py [cfg3] [segments] > profiles/<round>_restart_sweep.md
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import hashlib  # noqa: E402

import numpy as np  # noqa: E402
import torch  # noqa: E402

import ctypes  # noqa: E402

import paper_conf_ppopp_wintermzss19_b200 as acs  # noqa: E402
from paper_conf_ppopp_wintermzss19_b200 import _lib, api  # noqa: E402
from synth import config  # noqa: E402


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg3"
    nseg = int(sys.argv[2]) if len(sys.argv) > 2 else 64
    # keep the stream-ordered pool's freed memory cached between calls (the API allocates C
    # with cudaMallocAsync per call; without this each call re-maps gigabytes)
    try:
        cudart = ctypes.CDLL("libcudart.so.12")
        pool = ctypes.c_void_p()
        cudart.cudaDeviceGetDefaultMemPool(ctypes.byref(pool), 0)
        thr = ctypes.c_uint64(2 ** 64 - 1)
        cudart.cudaMemPoolSetAttribute(pool, 4, ctypes.byref(thr))   # cudaMemPoolAttrReleaseThreshold
    except OSError:
        pass
    A, B = config(cfg)
    dA = acs.DeviceCSR.from_host(A, "cuda")
    dB = dA if cfg != "cfg5" else acs.DeviceCSR.from_host(B, "cuda")
    plan = acs.Plan(num_segments=nseg)
    plan.multiply(dA, dB)
    torch.cuda.synchronize()
    pool = plan.info()["pool_bytes"]
    plan.close()
    print(f"# Restart sweep ({cfg}, fp64, {nseg} canonical segments; exact pool bound {pool / 1e6:.0f} MB)\n")
    print("| budget (fraction of the exact bound) | pieces | restarts | ms (the C call, synchronised, median of 5; C on the device) | vs one piece | C digest |")
    print("|---|---|---|---|---|---|")
    base = None
    a, b = api._csr_in(dA), api._csr_in(dB)
    st = api._stream_ptr(None)
    for frac in (1.0, 0.5, 0.33, 0.2, 0.1, 0.05, 0.03):
        bp = acs.Plan(num_segments=nseg, pool_limit_bytes=int(pool * frac) + 1)
        (rp, col, val), pieces, restarts = bp.multiply_budget(dA, dB)     # warm-up + result
        reps, t, ts = 5, 0.0, []
        for _ in range(reps):                            # the C call only (C stays on the device)
            c = _lib.CsrOut()
            npc, nrs = ctypes.c_int(0), ctypes.c_int(0)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            _lib.check(bp._lib.acspgemm_multiply_budget(bp._h, ctypes.byref(a), ctypes.byref(b), 1, st,
                                                        ctypes.byref(c), ctypes.byref(npc), ctypes.byref(nrs)),
                       "acspgemm_multiply_budget")
            ts.append(1e3 * (time.perf_counter() - t0))
            bp._lib.acspgemm_free_csr(ctypes.byref(c), st)
            torch.cuda.synchronize()
        ms = float(np.median(ts))
        print("<!-- reps ms: " + ", ".join(f"{x:.1f}" for x in ts) + " -->", flush=True)
        base = base or ms
        dig = hashlib.sha256(rp.tobytes() + col.tobytes() + val.tobytes()).hexdigest()[:16]
        print(f"| {frac:.2f} | {pieces} | {restarts} | {ms:.1f} | {ms / base:.2f}x | {dig} |", flush=True)
        bp.close()


if __name__ == "__main__":
    main()
