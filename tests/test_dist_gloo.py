"""Multi-process host logic of the row-segment multi-GPU driver on CPU (gloo,
world_size 2, 4 and 8 -- one canonical segment per rank at 8): canonical segments, per-rank ownership, (rows, nnz) all-gather
offsets, CSR broadcast and concatenation.  The per-rank multiply is the oracle here
(a CPU stand-in injected by the test; the product path itself has no CPU fallback)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import oracle
    from paper_conf_ppopp_wintermzss19_b200 import dist as adist
    from paper_conf_ppopp_wintermzss19_b200.api import DeviceCSR
    from synth import power_law_csr
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        A = power_law_csr(1500, 1500, mean_len=8, alpha=1.4, max_len=300, seed=4)

        def local(A_, B_, seg, s0, s1):
            return oracle.gustavson(A_, B_, row_begin=int(seg[s0]), row_end=int(seg[s1]))

        C, (roff, noff), offs = adist.dist_multiply(A, A, local_multiply=local)
        pieces = [None] * world
        dist.all_gather_object(pieces, (C.row_ptr, C.col, C.val))
        # broadcast of a CSR (CPU tensors stand in for device memory under gloo)
        M = None
        if rank == 0:
            M = DeviceCSR(A.rows, A.cols, torch.from_numpy(A.row_ptr.astype(np.int32)),
                          torch.from_numpy(A.col), torch.from_numpy(A.val))
        Mb = adist.broadcast_csr(M, torch.device("cpu"), torch.float64, src=0)
        ok_b = (Mb.rows == A.rows and (Mb.row_ptr.numpy() == A.row_ptr).all()
                and (Mb.col.numpy() == A.col).all() and (Mb.val.numpy() == A.val).all())
        if rank == 0:
            rp, col, val = adist.concat_pieces(pieces)
            full = oracle.gustavson(A, A)
            ok = ((rp == full.row_ptr).all() and (col == full.col).all()
                  and val.tobytes() == full.val.tobytes())
            # offsets agree with the concatenation
            ok_off = offs[0] == (0, 0) and all(
                offs[g][1] == int(sum(p[0][-1] for p in pieces[:g])) for g in range(world))
            q.put((bool(ok), bool(ok_off), bool(ok_b)))
        else:
            q.put((True, True, bool(ok_b)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4, 8])
def test_dist_multiply_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert all(p.exitcode == 0 for p in procs)
    assert all(all(r) for r in res), res


def test_rank_segments_and_offsets():
    from paper_conf_ppopp_wintermzss19_b200 import dist as adist
    from paper_conf_ppopp_wintermzss19_b200.segments import canonical_segments_host
    from oracle import alg
    assert [adist.rank_segments(8, 4, g) for g in range(4)] == [(0, 2), (2, 4), (4, 6), (6, 8)]
    assert adist.rank_segments(8, 1, 0) == (0, 8)
    with pytest.raises(ValueError):
        adist.rank_segments(8, 3, 0)
    assert adist.concat_offsets([5, 0, 7], [3, 2, 4]) == [(0, 0), (3, 5), (5, 5)]
    rng = np.random.default_rng(0)
    for _ in range(20):
        lens = rng.integers(0, 20, rng.integers(1, 300))
        rp = np.concatenate([[0], np.cumsum(lens)])
        assert canonical_segments_host(rp, 8) == alg.canonical_segments(rp, 8)
    seg = [0, 10, 25, 40]
    assert adist.local_segment_rows(seg, 1, 3) == [0, 15, 30]


def _rap_worker(rank, world, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import oracle
    from paper_conf_ppopp_wintermzss19_b200 import dist as adist
    from synth import aggregation_prolongator, poisson3d_7pt, transpose
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        n = 8
        A = poisson3d_7pt(n)
        P = aggregation_prolongator(n)
        R = transpose(P)

        def local(A_, B_, seg, s0, s1):
            return oracle.gustavson(A_, B_, row_begin=int(seg[s0]), row_end=int(seg[s1]))

        C, _, offs = adist.dist_rap(R, A, P, local_multiply=local)
        pieces = [None] * world
        dist.all_gather_object(pieces, (C.row_ptr, C.col, C.val))
        if rank == 0:
            rp, col, val = adist.concat_pieces(pieces)
            A4 = poisson3d_7pt(n // 2)       # R·A·P = 4·A7(n/2) (the closed form of the oracle tests)
            ok = ((rp == A4.row_ptr).all() and (col == A4.col).all() and (val == 4 * A4.val).all())
            q.put(bool(ok))
        else:
            q.put(True)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_dist_rap_gloo(world):
    """Distributed Galerkin product: A·P per rank, one all-gather of the
    A·P pieces, R·(A·P) per rank; the concatenation equals 4·A7(n/2) exactly."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rap_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert all(p.exitcode == 0 for p in procs)
    assert all(res), res
