"""GPU tests of the C-ABI behaviour beyond parity: error statuses, plan reuse, streams,
stage times, IEEE special values, empty inputs."""
import math

import numpy as np
import pytest
import torch

import oracle
from synth import CSR, from_coo, poisson2d_5pt, poisson3d_27pt, power_law_csr, random_csr

pytestmark = pytest.mark.gpu


def pkg():
    import paper_conf_ppopp_wintermzss19_b200 as p
    return p


def dev(M, dt=np.float64):
    return pkg().DeviceCSR.from_host(M, "cuda", dt)


def check(C, A, B, tol=1e-12):
    rp, col, val = C.to_numpy()
    ref = oracle.gustavson(A, B)
    assert (rp == ref.row_ptr).all() and (col == ref.col).all()
    assert (np.abs(val.astype(np.float64) - ref.val) <= tol * ref.absval).all()


def test_pool_limit_out_of_memory_then_recover(cuda_available):
    p = pkg()
    A = poisson3d_27pt(12)
    dA = dev(A)
    plan = p.Plan(pool_limit_bytes=1000)
    with pytest.raises(p.AcspgemmError) as ei:
        plan.multiply(dA, dA)
    assert ei.value.status == 4                      # ACSPGEMM_ERR_OUT_OF_MEMORY
    plan.close()
    plan = p.Plan()                                  # a fresh plan works
    check(plan.multiply(dA, dA), A, A)


def test_numeric_before_symbolic_is_not_ready(cuda_available):
    p = pkg()
    plan = p.Plan()
    t = torch.zeros(4, dtype=torch.int32, device="cuda")
    v = torch.zeros(4, dtype=torch.float64, device="cuda")
    with pytest.raises(p.AcspgemmError) as ei:
        plan.numeric(t, t, v)
    assert ei.value.status == 6                      # ACSPGEMM_ERR_NOT_READY


def test_plan_reuse_grow_and_shrink(cuda_available):
    p = pkg()
    plan = p.Plan()
    for A in (random_csr(50, 40, 0.1, seed=1), poisson3d_27pt(14), random_csr(300, 300, 0.02, seed=2),
              power_law_csr(2000, 2000, 10, 1.3, 800, seed=3), poisson2d_5pt(8)):
        B = A if A.rows == A.cols else random_csr(A.cols, 30, 0.2, seed=4)
        check(plan.multiply(dev(A), dev(B)), A, B)


def test_stage_times(cuda_available):
    p = pkg()
    A = power_law_csr(3000, 3000, 12, 1.2, 1500, seed=7)
    plan = p.Plan(stage_times=True)
    plan.multiply(dev(A), dev(A))
    torch.cuda.synchronize()
    st = plan.stage_times()
    assert list(st) == list(p.STAGES)
    assert all(v >= 0 for v in st.values()) and st["ESC"] > 0


def test_two_plans_two_streams(cuda_available):
    p = pkg()
    A1, A2 = poisson3d_27pt(16), power_law_csr(4000, 4000, 10, 1.3, 1000, seed=11)
    d1, d2 = dev(A1), dev(A2)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    p1, p2 = p.Plan(), p.Plan()
    torch.cuda.synchronize()
    with torch.cuda.stream(s1):
        C1 = p1.multiply(d1, d1, s1)
    with torch.cuda.stream(s2):
        C2 = p2.multiply(d2, d2, s2)
    torch.cuda.synchronize()
    check(C1, A1, A1)
    check(C2, A2, A2)


def test_ieee_special_values(cuda_available):
    """NaN and Inf propagate (no fast-math, reading R22): entries whose sum involves a
    NaN are NaN, Inf·0 gives NaN, finite entries match the oracle."""
    A = from_coo(3, 3, [0, 0, 1, 2], [0, 1, 1, 2], np.array([np.nan, 1.0, np.inf, 2.0]))
    B = from_coo(3, 3, [0, 1, 1, 2], [0, 0, 2, 2], np.array([1.0, 3.0, 0.0, 5.0]))
    C = pkg().multiply(dev(A), dev(B))
    rp, col, val = C.to_numpy()
    ref = oracle.gustavson(A, B)
    assert (rp == ref.row_ptr).all() and (col == ref.col).all()
    for g, r in zip(val, ref.val):
        assert (math.isnan(g) and math.isnan(r)) or g == r


def test_empty_inputs(cuda_available):
    p = pkg()
    Z = CSR(0, 5, np.zeros(1, np.int32), np.zeros(0, np.int32), np.zeros(0))
    B = random_csr(5, 6, 0.5, seed=1)
    C = p.multiply(dev(Z), dev(B))
    assert C.rows == 0 and C.nnz == 0
    Zr = random_csr(7, 5, 0.0, seed=2)
    C = p.multiply(dev(Zr), dev(B))
    rp, _, _ = C.to_numpy()
    assert C.nnz == 0 and (rp == 0).all() and rp.shape[0] == 8
    rp, col, val = p.multiply_lib_alloc(dev(Zr), dev(B))
    assert rp.shape[0] == 8 and (rp == 0).all() and col.size == 0


def test_fp32_accumulates_in_fp32(cuda_available):
    """fp32 inputs accumulate in fp32 (reading R14): a row whose exact sum needs more than
    24 bits differs from the fp64 oracle by at most the fp32 tolerance."""
    n = 3000
    A = from_coo(1, n, np.zeros(n), np.arange(n), np.full(n, 1.0 + 2.0 ** -20))
    B = from_coo(n, 1, np.arange(n), np.zeros(n), np.full(n, 1.0 + 2.0 ** -21))
    C = pkg().multiply(dev(A, np.float32), dev(B, np.float32))
    _, _, val = C.to_numpy()
    ref = oracle.gustavson(A.astype(np.float32), B.astype(np.float32))
    assert val.dtype == np.float32
    assert abs(float(val[0]) - ref.val[0]) <= 1e-5 * ref.absval[0]


def test_binding_argument_checks(cuda_available):
    p = pkg()
    A = dev(random_csr(5, 5, 0.5, seed=3))
    Af = dev(random_csr(5, 5, 0.5, seed=3), np.float32)
    with pytest.raises(TypeError):
        p.multiply(A, Af)
    cpuA = p.DeviceCSR(A.rows, A.cols, A.row_ptr.cpu(), A.col.cpu(), A.val.cpu())
    with pytest.raises(ValueError):
        p.multiply(cpuA, cpuA)


def test_segment_options(cuda_available):
    """num_segments out of range and malformed explicit segments are rejected; any valid
    segmentation gives a correct C (bits may differ from the canonical 8-segment one)."""
    p = pkg()
    with pytest.raises(p.AcspgemmError):
        p.Plan(num_segments=65)
    A = power_law_csr(3000, 3000, 10, 1.3, 900, seed=21)
    dA = dev(A)
    plan = p.Plan()
    with pytest.raises(p.AcspgemmError):
        plan.set_segments([5, 100, A.rows])               # must start at row 0
    with pytest.raises(p.AcspgemmError):
        plan.set_segments([0, 2000, 1000, A.rows])        # must be non-decreasing
    for segs in ([0, A.rows], [0, 1000, 1000, 2999, A.rows], None):
        plan.set_segments(segs)
        check(plan.multiply(dA, dA), A, A)
    for S in (1, 3, 64):
        check(p.multiply(dA, dA, num_segments=S), A, A)


def test_fp32_bit_identical_across_segment_splits(cuda_available):
    p = pkg()
    A = power_law_csr(4000, 4000, 10, 1.3, 1200, seed=23)
    dA = dev(A, np.float32)
    full = p.multiply(dA, dA)
    frp, fcol, fval = full.to_numpy()
    seg = p.canonical_segments(dA, 8)
    pieces = []
    for g in range(4):
        r0, r1 = seg[2 * g], seg[2 * g + 2]
        plan = p.Plan()
        plan.set_segments([r - r0 for r in seg[2 * g:2 * g + 3]])
        view = p.api._csr_in(dA, row_ptr=dA.row_ptr[r0:r1 + 1], rows=r1 - r0,
                             nnz=int(A.row_ptr[r1] - A.row_ptr[r0]))
        pieces.append(plan.multiply(dA, dA, A_view=view).to_numpy())
    from paper_conf_ppopp_wintermzss19_b200.dist import concat_pieces
    rp, col, val = concat_pieces(pieces)
    assert (rp == frp).all() and (col == fcol).all() and val.tobytes() == fval.tobytes()


def test_rap_galerkin(cuda_available):
    """acspgemm_rap / rap: R·(A·P) = 4·A₇(n/2) exactly for 2³ aggregation (§8(f)-2)."""
    from synth import aggregation_prolongator, poisson3d_7pt, transpose
    p = pkg()
    n = 16
    A, P = poisson3d_7pt(n), aggregation_prolongator(n)
    R = transpose(P)
    A4 = poisson3d_7pt(n // 2)
    C = p.rap(dev(R), dev(A), dev(P))
    rp, col, val = C.to_numpy()
    assert (rp == A4.row_ptr).all() and (col == A4.col).all() and (val == 4 * A4.val).all()
    rp, col, val = p.rap_lib_alloc(dev(R), dev(A), dev(P))
    assert (rp == A4.row_ptr).all() and (col == A4.col).all() and (val == 4 * A4.val).all()


@pytest.mark.parametrize("pieces", [1, 3, 8])
def test_multiply_host_pieces_bit_identical(pieces, cuda_available):
    """acspgemm_multiply_host: host in, host out, pipelined over canonical-segment pieces;
    C equals the device multiply byte for byte and the oracle within tolerance."""
    p = pkg()
    A = power_law_csr(4000, 4000, 10, 1.3, 1200, seed=31)
    full = p.multiply(dev(A), dev(A))
    frp, fcol, fval = full.to_numpy()
    rp, col, val = p.multiply_host(A, A, pieces=pieces)
    assert (rp.numpy() == frp).all() and (col.numpy() == fcol).all()
    assert val.numpy().tobytes() == fval.tobytes()
    ref = oracle.gustavson(A, A)
    assert (np.abs(val.numpy() - ref.val) <= 1e-12 * ref.absval).all()


@pytest.mark.parametrize("pieces", [2, 8])
def test_multiply_host_banded_inputs_in_pieces(pieces, cuda_available):
    """B is A and banded: a piece waits only for the input pieces holding the rows its
    entries reach (their column range, read back per piece), the later pieces' copies
    still in flight -- C equals the device multiply byte for byte."""
    from synth import poisson3d_27pt
    p = pkg()
    A = poisson3d_27pt(24)
    full = p.multiply(dev(A), dev(A))
    frp, fcol, fval = full.to_numpy()
    rp, col, val = p.multiply_host(A, A, pieces=pieces)
    assert (rp.numpy() == frp).all() and (col.numpy() == fcol).all()
    assert val.numpy().tobytes() == fval.tobytes()


def test_multiply_host_rectangular_capacity(cuda_available):
    """B distinct from A (copied separately), numpy buffers, capacity overflow reports nnz."""
    p = pkg()
    A = random_csr(300, 500, 0.02, seed=41)
    B = random_csr(500, 200, 0.03, seed=42)
    ref = oracle.gustavson(A, B)
    nnz = int(ref.row_ptr[-1])
    plan = p.Plan()
    small = (np.zeros(301, np.int32), np.zeros(max(nnz - 1, 1), np.int32), np.zeros(max(nnz - 1, 1)))
    with pytest.raises(p.AcspgemmError):
        plan.multiply_host(A, B, out=small, pieces=2)
    out = (np.zeros(301, np.int32), np.zeros(nnz + 5, np.int32), np.zeros(nnz + 5))
    rp, col, val = plan.multiply_host(A, B, out=out, pieces=2)
    assert (rp == ref.row_ptr).all() and (col == ref.col).all()
    assert (np.abs(val - ref.val) <= 1e-12 * ref.absval).all()
    # the plan's own segmentation is restored afterwards
    check(plan.multiply(dev(A), dev(B)), A, B)


def test_sm_load_trace(cuda_available):
    """Table 3's lowest multiprocessor load (mpL, L760): with tracing on, every block a
    stage-2 kernel processed is recorded once (SM id, start, end); mpL is in (0, 1] for
    a kernel that ran on every SM, the per-SM busy times are non-negative, tracing
    changes no result, and an untraced plan reports NOT_READY."""
    import paper_conf_ppopp_wintermzss19_b200 as p
    from synth import poisson3d_27pt, power_law_csr
    A = poisson3d_27pt(40)
    dA = p.DeviceCSR.from_host(A, "cuda")
    plan = p.Plan()
    ref = plan.multiply(dA, dA)
    with pytest.raises(p.AcspgemmError):
        plan.sm_load("hash")
    plan.set_trace(True)
    C = plan.multiply(dA, dA)
    torch.cuda.synchronize()
    assert all(torch.equal(x, y) for x, y in ((C.row_ptr, ref.row_ptr), (C.col, ref.col), (C.val, ref.val)))
    info = plan.info()
    L = plan.sm_load("hash")
    assert L["blocks"] == info["nhash_blocks"] > 0
    assert 0.0 < L["mpl"] <= 1.0 and min(L["per_sm_ms"]) >= 0.0
    B = power_law_csr(3000, 3000, mean_len=12, alpha=1.3, max_len=800, seed=2)
    dB = p.DeviceCSR.from_host(B, "cuda")
    plan.multiply(dB, dB)
    E = plan.sm_load("esc")
    assert E["blocks"] > 0 and 0.0 <= E["mpl"] <= 1.0
    plan.set_trace(False)
    plan.multiply(dB, dB)
    with pytest.raises(p.AcspgemmError):
        plan.sm_load("esc")
    plan.close()


def test_plan_reuse_scan_state_many_tiles(cuda_available):
    """The one-pass scans keep a ticket, a done counter and per-tile posts in plan memory
    and leave them zero (scan.cu).  Alternate large (many tiles: 70,001 rows = 69 tiles
    of the row-pointer scan) and tiny multiplies on one plan, and a multiply with a
    capture in between (numeric_update), and check every C exactly."""
    p = pkg()
    plan = p.Plan()
    big = random_csr(70001, 70001, 4e-5, seed=31)
    mid = power_law_csr(9000, 9000, 6, 1.4, 3000, seed=32)
    tiny = poisson2d_5pt(3)
    for A in (big, tiny, mid, big, tiny, big):
        dA = dev(A)
        C = plan.multiply(dA, dA)
        check(C, A, A)
        if A is mid:
            s = torch.cuda.Stream()
            with torch.cuda.stream(s):
                plan.numeric_update(dA, dA, C, s)
            s.synchronize()
            check(C, A, A)
