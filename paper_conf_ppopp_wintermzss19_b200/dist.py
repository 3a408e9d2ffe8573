"""Multi-GPU driver: row-segment data parallelism (one process per GPU).

The paper is single-GPU.  The extension (reading R21):
A is cut into S = 8 canonical nnz-balanced row segments, independent of the GPU count;
rank g of G owns segments [g·S/G, (g+1)·S/G) and multiplies that row range of A with
the full B (broadcast over NCCL).  Because blocks are counted from each segment's first
nonzero and rows never cross segments, every block, chunk, merge and summation tree is
the same for every G: the concatenated C is byte-identical to the 1-GPU result.
C stays distributed as CSR pieces; `gather_offsets` gives each piece's row and nnz offset
(an all-gather of one int64 per rank).

Host logic only; every multiply runs through the C ABI (`Plan.multiply` with a row-range
view of A).
"""
from __future__ import annotations

from typing import Callable, List, Optional, Sequence, Tuple

import torch
import torch.distributed as dist

S_DEFAULT = 8


def rank_segments(S: int, G: int, g: int) -> Tuple[int, int]:
    """Segments [s0, s1) owned by rank g of G (G must divide S)."""
    if S % G:
        raise ValueError(f"the GPU count ({G}) must divide the segment count ({S})")
    return g * S // G, (g + 1) * S // G


def local_segment_rows(seg: Sequence[int], s0: int, s1: int) -> List[int]:
    """Segment boundaries of the rank's row range, relative to its first row."""
    r0 = seg[s0]
    return [int(r) - int(r0) for r in seg[s0:s1 + 1]]


def concat_offsets(local_nnz: Sequence[int], local_rows: Sequence[int]) -> List[Tuple[int, int]]:
    """(row offset, nnz offset) of each rank's piece in the concatenated C."""
    out, r, n = [], 0, 0
    for rows, nnz in zip(local_rows, local_nnz):
        out.append((r, n))
        r += int(rows)
        n += int(nnz)
    return out


def gather_offsets(local_nnz: int, local_rows: int, group=None, device=None) -> List[Tuple[int, int]]:
    """all_gather of (rows, nnz) per rank -> concat_offsets."""
    ws = dist.get_world_size(group)
    t = torch.tensor([local_rows, local_nnz], dtype=torch.int64, device=device)
    outs = [torch.zeros_like(t) for _ in range(ws)]
    dist.all_gather(outs, t, group=group)
    rows = [int(o[0].item()) for o in outs]
    nnz = [int(o[1].item()) for o in outs]
    return concat_offsets(nnz, rows)


def concat_pieces(pieces):
    """Concatenate per-rank CSR pieces (row_ptr, col, val) as numpy/torch arrays."""
    import numpy as np
    rps, cols, vals = [], [], []
    off = 0
    for i, (rp, col, val) in enumerate(pieces):
        rp = np.asarray(rp, dtype=np.int64)
        rps.append(rp[(0 if i == 0 else 1):] + off)
        off += int(rp[-1])
        cols.append(np.asarray(col))
        vals.append(np.asarray(val))
    return np.concatenate(rps), np.concatenate(cols), np.concatenate(vals)


def broadcast_csr(M, device, val_dtype, src: int = 0, group=None):
    """Broadcast a DeviceCSR from `src` (None on the other ranks) over the process group."""
    from .api import DeviceCSR
    rank = dist.get_rank(group)
    hdr = torch.zeros(3, dtype=torch.int64, device=device)
    if rank == src:
        hdr[0], hdr[1], hdr[2] = M.rows, M.cols, M.nnz
    dist.broadcast(hdr, src=src, group=group)
    rows, cols, nnz = (int(x) for x in hdr.tolist())
    if rank == src:
        rp, col, val = M.row_ptr, M.col, M.val.to(val_dtype)
    else:
        rp = torch.empty(rows + 1, dtype=torch.int32, device=device)
        col = torch.empty(nnz, dtype=torch.int32, device=device)
        val = torch.empty(nnz, dtype=val_dtype, device=device)
    for t in (rp, col, val):
        dist.broadcast(t, src=src, group=group)
    return DeviceCSR(rows, cols, rp, col, val)


def segment_multiply(A, B, seg: Sequence[int], s0: int, s1: int, plan=None, stream=None):
    """C rows [seg[s0], seg[s1]) = A[rows]·B through the C ABI with explicit segments."""
    from . import api
    own = plan is None
    p = api.Plan() if own else plan
    try:
        r0, r1 = int(seg[s0]), int(seg[s1])
        p.set_segments(local_segment_rows(seg, s0, s1))
        rp_view = A.row_ptr[r0:r1 + 1]
        nnz = int(rp_view[-1].item() - rp_view[0].item()) if r1 > r0 else 0
        view = api._csr_in(A, row_ptr=rp_view, rows=r1 - r0, nnz=nnz)
        return p.multiply(A, B, stream, A_view=view)
    finally:
        if own:
            p.close()


def dist_multiply(A, B, group=None, S: int = S_DEFAULT,
                  local_multiply: Optional[Callable] = None):
    """C = A·B over the process group: this rank's piece plus (row, nnz) offsets.

    A and B must be present on every rank (see broadcast_csr).  `local_multiply(A, B,
    seg, s0, s1)` defaults to segment_multiply (the CUDA path); tests inject a CPU
    stand-in to exercise the host logic with gloo."""
    from . import api
    G = dist.get_world_size(group)
    g = dist.get_rank(group)
    seg = api.canonical_segments(A, S) if local_multiply is None else None
    if seg is None:
        from .segments import canonical_segments_host
        seg = canonical_segments_host(A.row_ptr, S)
    s0, s1 = rank_segments(S, G, g)
    fn = local_multiply or segment_multiply
    C = fn(A, B, seg, s0, s1)
    rows = int(seg[s1]) - int(seg[s0])
    nnz = int(C.nnz) if hasattr(C, "nnz") else int(C[0][-1])
    dev = None
    if dist.get_backend(group) == "nccl":
        dev = torch.device("cuda", torch.cuda.current_device())
    offs = gather_offsets(nnz, rows, group, dev)
    return C, offs[g], offs


def allgather_csr_pieces(piece, rows_total: int, cols: int, group=None):
    """The one exchange step of the distributed Galerkin product: every
    rank's CSR piece (row_ptr, col, val; numpy or torch) -> the concatenated matrix on
    every rank.  NCCL: device tensors padded to the largest piece; gloo: CPU objects."""
    import numpy as np
    from .api import DeviceCSR
    ws = dist.get_world_size(group)
    if dist.get_backend(group) != "nccl":
        allp = [None] * ws
        to_np = lambda t: t.cpu().numpy() if hasattr(t, "cpu") else np.asarray(t)   # noqa: E731
        dist.all_gather_object(allp, tuple(to_np(t) for t in piece), group=group)
        rp, col, val = concat_pieces(allp)
        return rp, col, val
    dev = torch.device("cuda", torch.cuda.current_device())
    rp, col, val = piece
    sizes = torch.tensor([rp.numel() - 1, col.numel()], dtype=torch.int64, device=dev)
    alls = [torch.zeros_like(sizes) for _ in range(ws)]
    dist.all_gather(alls, sizes, group=group)
    mr = max(int(a[0]) for a in alls)
    mn = max(int(a[1]) for a in alls)
    def gather(t, n, dtype):
        buf = torch.zeros(n, dtype=dtype, device=dev)
        buf[:t.numel()] = t
        outs = [torch.empty_like(buf) for _ in range(ws)]
        dist.all_gather(outs, buf, group=group)
        return outs
    rps = gather(rp.to(torch.int64), mr + 1, torch.int64)
    cols = gather(col, max(mn, 1), col.dtype)
    vals = gather(val, max(mn, 1), val.dtype)
    out_rp, out_c, out_v, off = [torch.zeros(1, dtype=torch.int64, device=dev)], [], [], 0
    for g in range(ws):
        r, n = int(alls[g][0]), int(alls[g][1])
        out_rp.append(rps[g][1:r + 1] - rps[g][0] + off)
        out_c.append(cols[g][:n])
        out_v.append(vals[g][:n])
        off += n
    full_rp = torch.cat(out_rp).to(torch.int32)
    assert full_rp.numel() == rows_total + 1
    return DeviceCSR(rows_total, cols, full_rp.contiguous(), torch.cat(out_c).contiguous(),
                     torch.cat(out_v).contiguous())


def dist_rap(R, A, P, group=None, S: int = S_DEFAULT, local_multiply: Optional[Callable] = None):
    """Galerkin product R·(A·P) over the process group.

    Step 1: each rank multiplies its canonical segments of A's fine rows with P (no
    exchange: P is replicated).  Step 2: one all-gather of the A·P pieces -- R's coarse
    rows reach fine rows of every segment.  Step 3: each rank multiplies its canonical
    segments of R with the gathered A·P.  Both products use canonical segments, so the
    concatenated result is byte-identical to the 1-GPU R·(A·P) (acspgemm_rap).
    Returns (this rank's piece of R·A·P, its (row, nnz) offset, all offsets)."""
    AP_piece, _, _ = dist_multiply(A, P, group, S, local_multiply)
    AP = allgather_csr_pieces((AP_piece.row_ptr, AP_piece.col, AP_piece.val), A.rows, P.cols, group)
    if isinstance(AP, tuple):                      # gloo: the gathered A·P arrives on the host
        rp, col, val = AP
        if local_multiply is None:                 # the CUDA path: back to the device
            from .api import DeviceCSR
            dev = torch.device("cuda", torch.cuda.current_device())
            AP = DeviceCSR(A.rows, P.cols, torch.from_numpy(rp.astype("int32")).to(dev),
                           torch.from_numpy(col).to(dev), torch.from_numpy(val).to(dev))
        else:                                      # a CPU stand-in multiply (tests)
            from types import SimpleNamespace
            AP = SimpleNamespace(rows=A.rows, cols=P.cols, row_ptr=rp, col=col, val=val)
    return dist_multiply(R, AP, group, S, local_multiply)
