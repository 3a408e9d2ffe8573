"""The multi-GPU driver's CUDA path on one GPU: distributed multiply and
the distributed Galerkin product R·(A·P) (one all-gather of the A·P pieces) with a
one-rank gloo group, byte for byte against the single-plan results; and the one-GPU
strong-scaling proxy's pieces (a rank's share of the canonical segments) concatenating to
the full C."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist

from synth import aggregation_prolongator, poisson3d_27pt, poisson3d_7pt, transpose

pytestmark = pytest.mark.gpu


def pkg():
    import paper_conf_ppopp_wintermzss19_b200 as p
    return p


@pytest.fixture
def group1():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1)
    yield
    dist.destroy_process_group()


def dev_csr(M, dt=np.float64):
    return pkg().DeviceCSR.from_host(M, "cuda", dt)


def same(C, D):
    return all(torch.equal(a.cpu(), b.cpu()) for a, b in ((C.row_ptr, D.row_ptr), (C.col, D.col), (C.val, D.val)))


def test_dist_rap_matches_rap(group1, cuda_available):
    from paper_conf_ppopp_wintermzss19_b200 import dist as adist
    n = 32
    A, P = poisson3d_7pt(n), aggregation_prolongator(n)
    R = transpose(P)
    dR, dA, dP = dev_csr(R), dev_csr(A), dev_csr(P)
    C, off, offs = adist.dist_rap(dR, dA, dP)
    ref = pkg().rap(dR, dA, dP)
    torch.cuda.synchronize()
    assert off == (0, 0) and same(C, ref)
    A4 = poisson3d_7pt(n // 2)
    assert (C.val.cpu().numpy() == 4 * A4.val).all()


def test_segment_shares_concatenate(cuda_available):
    """A rank's share (segments [g·8/N, (g+1)·8/N)) multiplied alone, for N = 2, 4, 8:
    the pieces concatenate to the single-plan C byte for byte (what bench.py and the
    scaling proxy time per rank)."""
    from paper_conf_ppopp_wintermzss19_b200 import dist as adist
    A = poisson3d_27pt(20)
    A.val[:] = np.random.default_rng(3).uniform(-1, 1, A.val.shape)
    dA = dev_csr(A)
    ref = pkg().multiply(dA, dA)
    seg = pkg().canonical_segments(dA, 8)
    for N in (2, 4, 8):
        pieces = []
        for g in range(N):
            s0, s1 = adist.rank_segments(8, N, g)
            C = adist.segment_multiply(dA, dA, seg, s0, s1)
            pieces.append((C.row_ptr.cpu().numpy(), C.col.cpu().numpy(), C.val.cpu().numpy()))
        rp, col, val = adist.concat_pieces(pieces)
        assert (rp == ref.row_ptr.cpu().numpy()).all() and (col == ref.col.cpu().numpy()).all()
        assert val.tobytes() == ref.val.cpu().numpy().tobytes()
