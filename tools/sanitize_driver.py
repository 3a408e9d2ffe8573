"""Small multiplies that reach every kernel of the library, for compute-sanitizer
(memcheck, racecheck, synccheck, initcheck on small configs).

usage: compute-sanitizer --tool TOOL python tools/sanitize_driver.py
Each case is also checked against the CPU oracle (structure exact, values within the
north-star tolerance), so a run prints one line per case and "sanitize-driver ok".
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ppopp_wintermzss19_b200 as acs  # noqa: E402
from synth import (aggregation_prolongator, from_coo, poisson2d_5pt, poisson3d_7pt, poisson3d_27pt,  # noqa: E402
                   power_law_csr, random_csr, random_rowlen_csr)

TOL = {np.float64: 1e-12, np.float32: 1e-5}


def case(name, A, B, dt, strategy="adaptive", index64=False):
    plan = acs.Plan(strategy=strategy, stage_times=True)
    dA = acs.DeviceCSR.from_host(A, "cuda", dt)
    dB = dA if B is A else acs.DeviceCSR.from_host(B, "cuda", dt)
    C = plan.multiply(dA, dB, index64=index64)
    torch.cuda.synchronize()
    rp, col, val = C.to_numpy()
    ref = oracle.gustavson(A.astype(dt), B.astype(dt))
    assert (rp == ref.row_ptr).all() and (col == ref.col).all(), name
    assert not (np.abs(val.astype(np.float64) - ref.val) > TOL[dt] * ref.absval).any(), name
    info = plan.info()
    plan.stage_times()
    plan.close()
    print(f"{name:28s} {np.dtype(dt).name:8s} {strategy:8s} nnz={len(col)} blocks={info['nblocks']} "
          f"dict={info['ndict_blocks']} hash={info['nhash_blocks']} path={info['npath']} search={info['nsearch']}",
          flush=True)


def main():
    rng = np.random.default_rng(5)
    s27 = poisson3d_27pt(10)
    s27.val[:] = rng.uniform(-1, 1, s27.val.shape)
    case("27pt dict", s27, s27, np.float32)
    case("27pt hash", s27, s27, np.float64)
    case("27pt dict fp64", s27, s27, np.float64, "dict")
    case("27pt esc", s27, s27, np.float64, "esc")
    case("27pt index64", s27, s27, np.float64, "adaptive", True)
    case("5pt (esc, short B rows)", poisson2d_5pt(20), poisson2d_5pt(20), np.float64)
    case("A*P (small tiles)", poisson3d_7pt(8), aggregation_prolongator(8), np.float64)
    A = power_law_csr(1500, 1500, mean_len=12, alpha=1.2, max_len=900, seed=3)
    B = power_law_csr(1500, 1500, mean_len=12, alpha=1.2, max_len=1500, seed=13)
    case("power law (path/search)", A, B, np.float64)
    case("power law fp32", A, B, np.float32)
    n = 20000
    Ad = from_coo(2, n, [0] * 1000 + [1] * 5, list(range(0, n, 20)) + [1, 2, 3, 4, 5], np.ones(1005))
    Bd = random_rowlen_csr(n, n, np.full(n, 30), seed=3, values="int")
    case("dense row (search merge)", Ad, Bd, np.float64)
    n_b = 40000
    Ag = from_coo(3, n_b, [0] * n_b + [1, 1], list(range(n_b)) + [5, 9], rng.uniform(-1, 1, n_b + 2))
    Bg = random_rowlen_csr(n_b, 100000, np.full(n_b, 32), seed=18, values="uniform")
    case("giant row (dense slices)", Ag, Bg, np.float64)
    # long B rows (> CAP entries): long-row chunks (R35) between short entries
    nb = 120
    blen = rng.integers(5, 40, nb)
    blen[::7] = rng.integers(2100, 3000, len(blen[::7]))
    Bl = random_rowlen_csr(nb, 4000, blen, seed=21)
    Al = random_rowlen_csr(600, nb, rng.integers(1, 10, 600), seed=22)
    case("long B rows (long-row chunks)", Al, Bl, np.float64)
    # LP-like: rows of ~1,600 products (no kept row, R38; two-chunk rows > 512: Multi Merge)
    from synth import lp_like
    Alp, Atp = lp_like(rows_log2=11, cols_log2=13, per_col=20, seed=7)
    case("LP-like (Multi Merge)", Alp, Atp, np.float64)
    plan = acs.Plan()
    plan.set_trace(True)
    dT = acs.DeviceCSR.from_host(s27, "cuda")
    plan.multiply(dT, dT)
    torch.cuda.synchronize()
    assert plan.sm_load("hash")["blocks"] > 0
    plan.close()
    print("traced multiply (mpL) ok", flush=True)
    Ar, Br = random_csr(800, 700, 0.02, seed=1), random_csr(700, 900, 0.02, seed=2)
    case("random", Ar, Br, np.float32)
    Ae = from_coo(4, 6, [], [], [])
    case("empty", Ae, random_csr(6, 5, 0.5, seed=4), np.float64)
    # host-in / host-out pieces (the bench's e2e API), 4 row pieces
    plan = acs.Plan()
    A64 = s27.astype(np.float64)
    rp, col, val = plan.multiply_host(A64, A64, pieces=4)
    plan.close()
    ref = oracle.gustavson(A64, A64)
    assert (np.asarray(rp) == ref.row_ptr).all() and (np.asarray(col) == ref.col).all()
    assert not (np.abs(np.asarray(val) - ref.val) > 1e-12 * ref.absval).any()
    print("multiply_host pieces=4 ok", flush=True)
    print("sanitize-driver ok")


if __name__ == "__main__":
    main()
