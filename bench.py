"""AC-SpGEMM benchmark (driver contract: one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl cuda|reference]
                    [--config cfg2] [--dtype f64|f32] [--no-cpu-baseline] [--no-e2e]

A "step" is one complete C = A·B through the C ABI (symbolic: GLB, AC-ESC, MCC,
merges, row_ptr scan; torch allocation of C; numeric: chunk copy) on inputs resident in
HBM.  The default workload is BASELINE.json configs[1]: C = A·A for the 3D 27-point
Poisson operator on a 128³ grid (2,097,152 rows, 55,742,968 nnz), fp64.  Inputs
(0.67 GB) and chunk pool (17.9 GB) are larger than the 126 MB L2, so no flush is needed.

Multi-GPU (torchrun, one process per GPU): A is broadcast from rank 0 over NCCL (timed
separately, not part of `value`), rank g runs canonical segments [g·8/N, (g+1)·8/N)
of A against the full B = A; per-rank nnz are all-gathered for the row_ptr offsets.
`value` = 2 × (products over all ranks) / max-over-ranks step time.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "SpGEMM GFLOPS (2x products / device time)"
UNIT = "GFLOP/s"
CONFIGS = {
    "cfg1": "C=A·A, 2D 5-point Poisson 64x64 (4,096 rows)",
    "cfg2": "C=A·A, 3D 27-point Poisson 128^3 (2,097,152 rows, 55,742,968 nnz)",
    "cfg3": "C=A·A, R-MAT scale 20 ef 16 (a,b,c,d=.45,.15,.15,.25)",
    "cfg5": "C=A·A^T, LP-like 2^20 x 2^22, 20 nnz/col",
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="cuda", choices=["cuda", "reference"])
    ap.add_argument("--config", default="cfg2", choices=sorted(CONFIGS))
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-pieces", type=int, default=8,
                    help="row pieces of acspgemm_multiply_host (copy-out overlaps the next piece)")
    ap.add_argument("--cpu-seconds", type=float, default=12.0, help="target CPU time of the oracle sample")
    return ap.parse_args()


def load_inputs(cfg: str, dt):
    from synth import config
    A, B = config(cfg, dt)
    return A.astype(dt), B.astype(dt)


# ------------------------------------------------------------------ clocks --

class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    def __init__(self, dev_index: int):
        self.dev = dev_index
        self.proc = None
        self.lines = []
        self.thread = None

    def start(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.dev), f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
            return
        def reader():
            for line in self.proc.stdout:
                self.lines.append(line.strip())
        self.thread = threading.Thread(target=reader, daemon=True)
        self.thread.start()
        t0 = time.time()
        while not self.lines and time.time() - t0 < 5.0:   # first sample before timing starts
            time.sleep(0.02)

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        if self.thread:
            self.thread.join(timeout=1)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 8:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[4:8]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ----------------------------------------------------------------- oracle --

def cpu_oracle_sample(A, B, target_s: float):
    """Time the oracle (as it stands) on rows [0, R) of A·B, R sized for ~target_s."""
    import oracle
    nthr = oracle.max_threads()
    rows = A.rows
    r = max(1, rows // 512)
    C, t = oracle.timed_gustavson(A, B, row_end=r)
    while t < 0.5 and r < rows:
        r = min(rows, r * 4)
        C, t = oracle.timed_gustavson(A, B, row_end=r)
    r = min(rows, max(1, int(r * target_s / max(t, 1e-6))))
    C, t = oracle.timed_gustavson(A, B, row_end=r)
    sub = type(A)(r, A.cols, A.row_ptr[:r + 1], A.col, A.val)
    prods = oracle.products(sub, B)
    return {"value": 2.0 * prods / t / 1e9, "unit": UNIT, "cores": nthr, "kind": "oracle",
            "sample": f"rows 0..{r} of {rows} ({prods} of the workload's products, {C.nnz} nnz of C), "
                      f"{t:.2f} s, fp64 SPA Gustavson, OpenMP static over rows"}, r


def run_reference(args):
    """--impl reference: the oracle on the box's host cores, bounded sample per step."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    dt = np.float64 if args.dtype == "f64" else np.float32
    A, B = load_inputs(args.config, dt)
    nthr = oracle.max_threads()
    per_step = max(0.5, min(8.0, 150.0 / max(1, args.steps + args.warmup)))
    base, r = cpu_oracle_sample(A, B, per_step)
    sub = type(A)(r, A.cols, A.row_ptr[:r + 1], A.col, A.val)
    prods = oracle.products(sub, B)
    for _ in range(args.warmup):
        oracle.gustavson(A, B, row_end=r)
    times = []
    for _ in range(args.steps):
        _, t = oracle.timed_gustavson(A, B, row_end=r)
        times.append(t)
    t = sum(times) / len(times)
    val = 2.0 * prods / t / 1e9
    out = {"metric": METRIC, "value": val, "unit": UNIT, "impl": "reference", "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
           "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
           "config": {"workload": args.config, "description": CONFIGS[args.config], "dtype": args.dtype,
                      "sample_rows": r, "rows": A.rows},
           "cpu_baseline": {"value": val, "unit": UNIT, "cores": nthr, "kind": "oracle",
                            "sample": f"rows 0..{r} of {A.rows} per step ({prods} products)"},
           "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)
    return 0


# ------------------------------------------------------------------- cuda --

def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_wintermzss19_b200 as acs
    from paper_conf_ppopp_wintermzss19_b200 import dist as adist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        args.gpus = world
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    dt = np.float64 if args.dtype == "f64" else np.float32
    tdt = torch.float64 if args.dtype == "f64" else torch.float32
    vbytes = 8 if args.dtype == "f64" else 4

    # ---- inputs: rank 0 builds A; broadcast over NCCL (timed separately) ----
    A = B = None
    if rank == 0:
        A, B = load_inputs(args.config, dt)
    t_bcast = None
    if world > 1:
        t0 = time.perf_counter()
        dA = adist.broadcast_csr(acs.DeviceCSR.from_host(A, dev) if rank == 0 else None, dev, tdt, src=0)
        same = args.config != "cfg5"
        dB = dA if same else adist.broadcast_csr(acs.DeviceCSR.from_host(B, dev) if rank == 0 else None, dev, tdt, 0)
        torch.cuda.synchronize()
        t_bcast = time.perf_counter() - t0
    else:
        dA = acs.DeviceCSR.from_host(A, dev)
        dB = dA if args.config != "cfg5" else acs.DeviceCSR.from_host(B, dev)

    # ---- this rank's canonical segments ----
    seg = acs.canonical_segments(dA, 8)
    s0, s1 = adist.rank_segments(8, world, rank)
    r0, r1 = seg[s0], seg[s1]
    plan = acs.Plan(stage_times=True)
    plan.set_segments([r - r0 for r in seg[s0:s1 + 1]])
    rp_view = dA.row_ptr[r0:r1 + 1]
    nnz_view = int(rp_view[-1].item() - rp_view[0].item())
    view = acs.api._csr_in(dA, row_ptr=rp_view, rows=r1 - r0, nnz=nnz_view)
    stream = torch.cuda.current_stream()

    def step():
        C = plan.multiply(dA, dB, stream, A_view=view)
        if world > 1:
            # the distributed C: per-rank pieces concatenated with row_ptr offsets, one
            # all-gather of (rows, nnz) per rank
            adist.gather_offsets(C.nnz, C.rows, device=dev)
        return C

    def digest(C, nnz_off):
        # order-independent 64-bit sums of row_ptr (offset to the concatenated C, without
        # the leading 0), column indices and value bits: equal for any GPU count
        s_rp = int((C.row_ptr[1:].to(torch.int64) + nnz_off).sum().item())
        s_col = int(C.col.to(torch.int64).sum().item())
        vb = C.val.view(torch.int64) if C.val.dtype == torch.float64 else C.val.view(torch.int32).to(torch.int64)
        s_val = int(vb.sum().item())
        t = torch.tensor([s_rp, s_col, s_val], dtype=torch.int64, device=dev)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.SUM)
        return "%016x-%016x-%016x" % tuple(int(x) & 0xFFFFFFFFFFFFFFFF for x in t.tolist())

    for _ in range(max(args.warmup, 0)):
        C = step()
        del C
    torch.cuda.synchronize()
    info = plan.info()

    # ---- timed region ----
    sampler = ClockSampler(local)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    esc_ms, hash_ms, dict_ms, stage_sum = [], [], [], {k: 0.0 for k in acs.STAGES}
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    sampler.start()
    ev0.record(stream)
    for _ in range(args.steps):
        C = step()
        st = plan.stage_times()
        esc_ms.append(st["ESC"])
        hash_ms.append(st["HASH"])
        dict_ms.append(st["DICT"])
        for k in st:
            stage_sum[k] += st[k]
        del C
    ev1.record(stream)
    torch.cuda.synchronize()
    clocks = sampler.stop()
    if world > 1:
        dist.barrier()
    ms_total = ev0.elapsed_time(ev1)
    ms_step = ms_total / max(args.steps, 1)
    products = info["products"]
    if world > 1:
        tt = torch.tensor([ms_step], dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms_step_max = float(tt.item())
        pp = torch.tensor([products], dtype=torch.int64, device=dev)
        dist.all_reduce(pp, op=dist.ReduceOp.SUM)
        products_all = int(pp.item())
    else:
        ms_step_max, products_all = ms_step, products
    value = 2.0 * products_all / (ms_step_max * 1e-3) / 1e9

    # ---- determinism digest of C (untimed) ----
    C = plan.multiply(dA, dB, stream, A_view=view)
    off = adist.gather_offsets(C.nnz, C.rows, device=dev)[rank][1] if world > 1 else 0
    c_digest = digest(C, off)
    del C

    # ---- roofline of the dominant kernel: the ESC stage runs k_dict then k_hash (adaptive
    # strategy, readings R33, R31) then k_esc on the blocks they left; the one holding most of the
    # stage is reported, timed live by the plan's CUDA events on the library stream ----
    esc_stage = sum(esc_ms) / len(esc_ms) if esc_ms else float("nan")
    hash_avg = sum(hash_ms) / len(hash_ms) if hash_ms else 0.0
    dict_avg = sum(dict_ms) / len(dict_ms) if dict_ms else 0.0
    if dict_avg >= 0.5 * esc_stage:
        kern, kern_tag, esc_avg = "k_dict", "dict", dict_avg
    elif hash_avg >= 0.5 * esc_stage:
        kern, kern_tag, esc_avg = "k_hash", "hash", hash_avg - dict_avg
    else:
        kern, kern_tag, esc_avg = "k_esc", "esc", esc_stage - hash_avg
    rows_b = dB.rows
    bytes_a = 4 * (view.rows + 1) + nnz_view * (4 + vbytes)
    bytes_b = 4 * (rows_b + 1) + dB.nnz * (4 + vbytes)
    bytes_chunks = info["chunk_elems"] * (4 + vbytes)
    esc_bytes = bytes_a + bytes_b + bytes_chunks
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    peak = float(peaks.get("hbm_gbs", 6650.0))
    peak_src = "measured" if "hbm_gbs" in peaks else "fallback"
    achieved = esc_bytes / (esc_avg * 1e-3) / 1e9
    traffic = None
    tf = os.path.join(ROOT, "profiles", f"{kern_tag}_traffic_{args.config}_{args.dtype}.json")
    if os.path.exists(tf):
        try:
            traffic = json.load(open(tf)).get("dram_bytes_per_launch")
        except Exception:
            traffic = None

    # ---- e2e through the public API with host buffers (rank-local) ----
    e2e = None
    if not args.no_e2e:
        e2e = measure_e2e(acs, torch, A, B, dA, dB, view, plan, dev, tdt, rank, world, r0, r1, args, products_all)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        try:
            cpu, _ = cpu_oracle_sample(A, B, args.cpu_seconds)
        except Exception as ex:  # never fail the bench line on the baseline
            cpu = {"value": None, "unit": UNIT, "cores": None, "kind": "oracle", "sample": f"failed: {ex}"}

    if rank == 0:
        out = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step_max, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            "config": {"workload": args.config, "description": CONFIGS[args.config],
                       "products": products_all, "nnz_c": info["nnz_c"] if world == 1 else None,
                       "l2": "inputs (A,B) and chunk pool exceed the 126 MB L2; no flush",
                       "parallelism": f"row-segments x{world}", "segments": 8},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "kernel": kern,
                         "algorithmic_bytes_per_launch": esc_bytes, "avg_launch_ms": esc_avg,
                         "peak_source": peak_src},
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": int(info["kernel_launches"]) * args.steps,
            "clocks": clocks,
            "stages_ms_per_step": {k: v / max(args.steps, 1) for k, v in stage_sum.items()},
            "plan": {k: info[k] for k in ("nblocks", "nchunks", "chunk_elems", "nshared", "nmulti", "npath",
                                          "nsearch", "merge_elems", "pool_bytes", "helper_bytes",
                                          "pool_estimate_bytes", "nhash_blocks", "ndict_blocks")},
            "strategy": "adaptive (hash accumulator per block, AC-ESC fallback; DESIGN R31)",
            "bcast_s": t_bcast,
            "c_digest": c_digest,
        }
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def measure_e2e(acs, torch, A, B, dA, dB, view, plan, dev, tdt, rank, world, r0, r1, args, products_all):
    """Same metric end to end: per step, H2D of this rank's inputs from pinned host
    memory, the multiply, and D2H of the result C into pinned host memory."""
    import torch.distributed as dist
    steps = max(1, min(args.steps, 5))
    if rank == 0 and A is not None:
        hA = [torch.from_numpy(np.ascontiguousarray(x)).pin_memory() for x in (A.row_ptr.astype(np.int32), A.col, A.val)]
        hB = None if args.config != "cfg5" else [torch.from_numpy(np.ascontiguousarray(x)).pin_memory()
                                                   for x in (B.row_ptr.astype(np.int32), B.col, B.val)]
    else:
        # other ranks copy their device inputs to pinned host once (the "user's" host data)
        hA = [t.cpu().pin_memory() for t in (dA.row_ptr, dA.col, dA.val)]
        hB = None if dB is dA else [t.cpu().pin_memory() for t in (dB.row_ptr, dB.col, dB.val)]
    if world == 1:
        return measure_e2e_host(acs, torch, A, B, hA, hB, plan, tdt, args, products_all)
    dA2 = acs.DeviceCSR(dA.rows, dA.cols, torch.empty_like(dA.row_ptr), torch.empty_like(dA.col), torch.empty_like(dA.val))
    dB2 = dA2 if hB is None else acs.DeviceCSR(dB.rows, dB.cols, torch.empty_like(dB.row_ptr),
                                               torch.empty_like(dB.col), torch.empty_like(dB.val))
    nnz_c = plan.info()["nnz_c"]
    h_rp = torch.empty(r1 - r0 + 1, dtype=torch.int32).pin_memory()
    h_col = torch.empty(max(nnz_c, 1), dtype=torch.int32).pin_memory()
    h_val = torch.empty(max(nnz_c, 1), dtype=tdt).pin_memory()
    stream = torch.cuda.current_stream()
    h2d = sum(t.numel() * t.element_size() for t in hA) + (0 if hB is None else sum(t.numel() * t.element_size() for t in hB))
    rp_view = dA2.row_ptr[r0:r1 + 1]
    view2 = acs.api._csr_in(dA2, row_ptr=rp_view, rows=view.rows, nnz=view.nnz)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    d2h = 0
    e0.record(stream)
    for _ in range(steps):
        for d, h in zip((dA2.row_ptr, dA2.col, dA2.val), hA):
            d.copy_(h, non_blocking=True)
        if hB is not None:
            for d, h in zip((dB2.row_ptr, dB2.col, dB2.val), hB):
                d.copy_(h, non_blocking=True)
        C = plan.multiply(dA2, dB2, stream, A_view=view2)
        n = C.nnz
        h_rp.copy_(C.row_ptr, non_blocking=True)
        h_col[:n].copy_(C.col, non_blocking=True)
        h_val[:n].copy_(C.val, non_blocking=True)
        d2h = h_rp.numel() * 4 + n * (4 + h_val.element_size())
        del C
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    if world > 1:
        tt = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms = float(tt.item())
    return {"value": 2.0 * products_all / (ms * 1e-3) / 1e9, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
            "d2h_bytes_per_step": int(d2h), "ms_per_step": ms, "steps": steps}


def measure_e2e_host(acs, torch, A, B, hA, hB, plan, tdt, args, products_all):
    """N = 1: the C-ABI host entry point acspgemm_multiply_host does the whole job per
    step -- A (and B) host->device from pinned memory, the multiply in --e2e-pieces row
    pieces, each piece's C device->host into pinned buffers while the next piece runs."""
    from types import SimpleNamespace
    steps = max(1, min(args.steps, 5))
    hAc = SimpleNamespace(rows=A.rows, cols=A.cols, row_ptr=hA[0], col=hA[1], val=hA[2])
    hBc = hAc if hB is None else SimpleNamespace(rows=B.rows, cols=B.cols, row_ptr=hB[0], col=hB[1], val=hB[2])
    nnz_c = plan.info()["nnz_c"]
    out = (torch.empty(A.rows + 1, dtype=torch.int32).pin_memory(), torch.empty(max(nnz_c, 1), dtype=torch.int32).pin_memory(),
           torch.empty(max(nnz_c, 1), dtype=tdt).pin_memory())
    plan.multiply_host(hAc, hBc, out=out, pieces=args.e2e_pieces)       # warm (allocator, pinned pages)
    stream = torch.cuda.current_stream()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(steps):
        rp, col, val = plan.multiply_host(hAc, hBc, out=out, pieces=args.e2e_pieces)
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    h2d = sum(t.numel() * t.element_size() for t in hA) + (0 if hB is None else sum(t.numel() * t.element_size() for t in hB))
    d2h = rp.numel() * 4 + col.numel() * (4 + val.element_size())
    return {"value": 2.0 * products_all / (ms * 1e-3) / 1e9, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
            "d2h_bytes_per_step": int(d2h), "ms_per_step": ms, "steps": steps,
            "api": f"acspgemm_multiply_host, {args.e2e_pieces} pieces"}


if __name__ == "__main__":
    sys.exit(main())
