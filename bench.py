"""AC-SpGEMM benchmark (driver contract: one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl cuda|reference]
                    [--config cfg2] [--dtype f64|f32] [--no-cpu-baseline] [--no-e2e]
                    [--no-side] [--backend nccl|gloo]

A "step" is one complete C = A·B through the C ABI (symbolic: GLB, AC-ESC / the adaptive
accumulators, MCC, merges, row_ptr scan; torch allocation of C; numeric: chunk copy) on
inputs resident in HBM.  The default workload is BASELINE.json configs[1]: C = A·A for
the 3D 27-point Poisson operator on a 128³ grid (2,097,152 rows, 55,742,968 nnz), fp64.
Inputs (0.67 GB) and chunk pool (~18 GB) are larger than the 126 MB L2, so no flush is
needed.

Reported besides the contract keys:
  * per-step median / min (CUDA events around every step) next to the K-step mean;
  * "method": the method bytes of one step -- |A| + |B| [+ products·(4+s) where B rows
    are reached randomly: cfg3, cfg5] + 3·nnz(C)·(4+s) + 4(rows+1) -- as GB/s and as a
    fraction of the measured HBM peak;
  * "roofline": the dominant kernel's algorithmic bytes per launch / its live duration;
  * "side": cfg3 and cfg5 in fp64, cfg2 in fp32 and cfg2 with the paper's pure AC-ESC
    strategy, each with GFLOPS, method fraction and its dominant kernel (N = 1 only);
  * "digest": SHA-256 of C per canonical segment (row lengths, columns, values),
    combined in segment order -- the same for every GPU count -- for the integer cfg2
    and for a U(-1,1)-valued cfg2 on the same pattern (which exposes any change of the
    summation order).

Multi-GPU (torchrun, one process per GPU): A is broadcast from rank 0 (timed separately,
not part of `value`), rank g runs canonical segments [g·8/N, (g+1)·8/N) of A against the
full B = A; per-rank nnz are all-gathered for the row_ptr offsets.  `value` = 2 ×
(products over all ranks) / max-over-ranks step time.  --backend gloo runs the N > 1 path
with gloo collectives (e.g. 2 ranks on one GPU for a dry run; NCCL refuses that).
"""
from __future__ import annotations

import argparse
import hashlib
import json
import os
import platform
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
RANDOM_B = {"cfg3", "cfg5"}            # B rows reached randomly: one B gather per product (§8(d))
L2_NOTE = "inputs (A,B) and chunk pool exceed the 126 MB L2; no flush"


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
    ap.add_argument("--no-side", action="store_true", help="skip the side workloads (cfg3, cfg5, cfg2 f32 / esc)")
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"])
    return ap.parse_args()


def products_of(A, B) -> int:
    """Intermediate products sum_k nnz(A_:,k) nnz(B_k,:) (numpy, from the inputs)."""
    blen = np.diff(np.asarray(B.row_ptr, dtype=np.int64))
    return int(blen[np.asarray(A.col, dtype=np.int64)].sum())


def config_dict(cfg: str, dtype: str, A, B, products: int) -> dict:
    """The workload description both arms print (identical dicts)."""
    return {"workload": cfg, "description": CONFIGS[cfg], "dtype": dtype, "rows": int(A.rows),
            "nnz_a": int(A.row_ptr[-1]), "products": int(products), "segments": 8, "l2": L2_NOTE}


def method_bytes(cfg: str, vbytes: int, rows_a: int, nnz_a: int, rows_b: int, nnz_b: int, products: int,
                 nnz_c: int) -> int:
    """|A| + |B| [+ products·(4+s) if random] + 3·nnz(C)(4+s) + 4(rows+1)."""
    e = 4 + vbytes
    a = 4 * (rows_a + 1) + nnz_a * e
    b = 4 * (rows_b + 1) + nnz_b * e
    g = products * e if cfg in RANDOM_B else 0
    return a + b + g + 3 * nnz_c * e + 4 * (rows_a + 1)


def cpu_model() -> str:
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return platform.processor() or "unknown"


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

def _sample_rows(A, B, target_s: float, threads: int = 0):
    """Rows [0, R) of A·B sized so the oracle (as it stands) takes ~target_s."""
    import oracle
    rows = A.rows
    r = max(1, rows // 512)
    C, t = oracle.timed_gustavson(A, B, threads=threads, row_end=r)
    while t < 0.5 and r < rows:
        r = min(rows, r * 4)
        C, t = oracle.timed_gustavson(A, B, threads=threads, row_end=r)
    r = min(rows, max(1, int(r * target_s / max(t, 1e-6))))
    C, t = oracle.timed_gustavson(A, B, threads=threads, row_end=r)
    sub = type(A)(r, A.cols, A.row_ptr[:r + 1], A.col, A.val)
    return r, C, t, products_of(sub, B)


def cpu_oracle_sample(A, B, target_s: float):
    """The oracle (fp64 SPA Gustavson, OpenMP static over rows) on the host cores, on a
    bounded row sample; plus a one-thread sample of ~target_s / 4."""
    import oracle
    nthr = oracle.max_threads()
    r, C, t, prods = _sample_rows(A, B, target_s)
    r1, _, t1, prods1 = _sample_rows(A, B, max(1.0, target_s / 4), threads=1)
    return {"value": 2.0 * prods / t / 1e9, "unit": UNIT, "cores": nthr, "kind": "oracle",
            "cpu_model": cpu_model(),
            "one_thread": {"value": 2.0 * prods1 / t1 / 1e9, "unit": UNIT, "sample_rows": r1, "seconds": t1},
            "sample": f"rows 0..{r} of {A.rows} ({prods} of the workload's products, {C.nnz} nnz of C), "
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
    r, _, _, prods = _sample_rows(A, B, per_step)
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
           "scaling": "weak" if args.gpus > 1 else "strong", "vs_baseline": None, "dtype": args.dtype,
           "data": "synthetic",
           "config": config_dict(args.config, args.dtype, A, B, products_of(A, B)),
           "cpu_baseline": {"value": val, "unit": UNIT, "cores": nthr, "kind": "oracle", "cpu_model": cpu_model(),
                            "sample": f"rows 0..{r} of {A.rows} per step ({prods} products), fp64 SPA Gustavson"},
           "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)
    return 0


# ------------------------------------------------------------------- cuda --

def timed_steps(torch, plan, dA, dB, view, stream, steps: int, warmup: int, stages, after=None):
    """W warm-up multiplies, then K timed ones: CUDA events around the K steps and around
    every step (median / min); the plan's stage times summed into `stages`.  `after(C)`
    runs inside each step (N > 1: the all-gather of the pieces' row / nnz offsets)."""
    for _ in range(max(warmup, 0)):
        C = plan.multiply(dA, dB, stream, A_view=view)
        del C
    torch.cuda.synchronize()
    E = torch.cuda.Event
    ev = [(E(enable_timing=True), E(enable_timing=True)) for _ in range(steps)]
    e0, e1 = E(enable_timing=True), E(enable_timing=True)
    per_stage = []
    e0.record(stream)
    for i in range(steps):
        ev[i][0].record(stream)
        C = plan.multiply(dA, dB, stream, A_view=view)
        if after is not None:
            after(C)
        ev[i][1].record(stream)
        st = plan.stage_times()
        per_stage.append(st)
        for k in st:
            stages[k] = stages.get(k, 0.0) + st[k]
        del C
    e1.record(stream)
    torch.cuda.synchronize()
    per = [a.elapsed_time(b) for a, b in ev]
    return e0.elapsed_time(e1), per, per_stage


def dominant_kernel(st_list):
    """The kernel holding most of the ESC stage (stage events): k_dict (DICT), k_hash
    (HASH - DICT) or AC-ESC with the per-row accumulator (ESC - HASH); its mean ms."""
    esc = statistics.mean(s["ESC"] for s in st_list)
    hsh = statistics.mean(s["HASH"] for s in st_list)
    dct = statistics.mean(s["DICT"] for s in st_list)
    if dct >= 0.5 * esc:
        return "k_dict", "dict", dct
    if hsh - dct >= 0.5 * esc:
        return "k_hash", "hash", hsh - dct
    return "k_esc", "esc", esc - hsh


def kernel_roofline(cfg, dtype, st_list, info, rows_a, nnz_a, rows_b, nnz_b, vbytes, peak, peak_src):
    kern, tag, ms = dominant_kernel(st_list)
    e = 4 + vbytes
    byts = 4 * (rows_a + 1) + nnz_a * e + 4 * (rows_b + 1) + nnz_b * e + info["chunk_elems"] * e
    if cfg in RANDOM_B:
        byts += info["products"] * e
    achieved = byts / (ms * 1e-3) / 1e9
    traffic = None
    issue = None
    tf = os.path.join(ROOT, "profiles", f"{tag}_traffic_{cfg}_{dtype}.json")
    if os.path.exists(tf):
        try:
            prof = json.load(open(tf))
            traffic = prof.get("dram_bytes_per_launch")
            inst = prof.get("metrics", {}).get("smsp__inst_executed.sum")
            if inst:
                # the issue-rate ceiling the counters show this kernel is near: warp
                # instructions per launch (committed ncu capture) over the live launch
                # time, against 4 schedulers x SMs x the max SM clock (one warp
                # instruction per scheduler per cycle)
                import torch
                sms = torch.cuda.get_device_properties(torch.cuda.current_device()).multi_processor_count
                mhz = float(os.environ.get("ACS_SM_MAX_MHZ", "1965"))
                ipk = inst / (ms * 1e-3) / 1e9
                pk = 4 * sms * mhz * 1e-3
                issue = {"achieved": ipk, "peak": pk, "unit": "G warp-instr/s", "frac": ipk / pk,
                         "warp_instr_per_launch": inst, "peak_source": f"4 x {sms} SMs x {mhz:.0f} MHz"}
        except Exception:
            traffic = None
    return {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
            "traffic": traffic, "kernel": kern, "algorithmic_bytes_per_launch": byts, "avg_launch_ms": ms,
            "peak_source": peak_src, "issue": issue}


def segment_digest(torch, C, seg_rows_local):
    """SHA-256 per canonical segment of a C piece (row lengths int32 | columns | values),
    combined in segment order: independent of how the segments are split over GPUs."""
    rp = C.row_ptr.to(torch.int64).cpu().numpy()
    col = C.col.cpu().numpy()
    val = C.val.cpu().numpy()
    out = []
    for s in range(len(seg_rows_local) - 1):
        a, b = seg_rows_local[s], seg_rows_local[s + 1]
        h = hashlib.sha256()
        h.update(np.diff(rp[a:b + 1]).astype(np.int32).tobytes())
        h.update(col[rp[a]:rp[b]].tobytes())
        h.update(val[rp[a]:rp[b]].tobytes())
        out.append(h.hexdigest())
    return out


def side_workloads(acs, torch, dev, peak, peak_src, dA2=None):
    """cfg3, cfg5 (fp64), cfg2 fp32 and cfg2 with the paper's pure AC-ESC strategy (fp64):
    5 timed multiplies each after 2 warm-ups (N = 1)."""
    out = {}
    stream = torch.cuda.current_stream()
    for name, cfg, dts, strategy in (("cfg3_f64", "cfg3", "f64", "adaptive"), ("cfg5_f64", "cfg5", "f64", "adaptive"),
                                     ("cfg2_f32", "cfg2", "f32", "adaptive"), ("cfg2_f64_esc", "cfg2", "f64", "esc")):
        try:
            dt = np.float64 if dts == "f64" else np.float32
            vbytes = 8 if dts == "f64" else 4
            if cfg == "cfg2" and dts == "f64" and dA2 is not None:
                dA = dB = dA2
                rows_a, nnz_a = dA.rows, dA.nnz
            else:
                A, B = load_inputs(cfg, dt)
                dA = acs.DeviceCSR.from_host(A, dev)
                dB = dA if cfg != "cfg5" else acs.DeviceCSR.from_host(B, dev)
                del A, B
            plan = acs.Plan(stage_times=True, strategy=strategy)
            tot, per, st = timed_steps(torch, plan, dA, dB, None, stream, 5, 2, {})
            info = plan.info()
            med = statistics.median(per)
            mb = method_bytes(cfg, vbytes, dA.rows, dA.nnz, dB.rows, dB.nnz, info["products"], info["nnz_c"])
            rl = kernel_roofline(cfg, dts, st, info, dA.rows, dA.nnz, dB.rows, dB.nnz, vbytes, peak, peak_src)
            out[name] = {"workload": cfg, "dtype": dts, "strategy": strategy, "ms_median": med, "ms_min": min(per),
                         "GFLOPS": 2.0 * info["products"] / (med * 1e-3) / 1e9,
                         "method_bytes": mb, "method_GBps": mb / (med * 1e-3) / 1e9,
                         "method_frac": mb / (med * 1e-3) / 1e9 / peak,
                         "kernel": rl["kernel"], "kernel_ms": rl["avg_launch_ms"], "kernel_frac": rl["frac"],
                         "stages_ms": {k: statistics.mean(s[k] for s in st) for k in st[0]},
                         "products": info["products"], "nnz_c": info["nnz_c"]}
            plan.close()
            del dA, dB
            torch.cuda.empty_cache()
        except Exception as ex:    # never fail the bench line on a side workload
            out[name] = {"error": str(ex)[:200]}
    return out


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
    ndev = max(1, torch.cuda.device_count())
    torch.cuda.set_device(local % ndev)
    dev = torch.device("cuda", local % ndev)
    if world > 1:
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
    cdev = dev if args.backend == "nccl" else torch.device("cpu")     # collectives' tensors
    dt = np.float64 if args.dtype == "f64" else np.float32
    tdt = torch.float64 if args.dtype == "f64" else torch.float32
    vbytes = 8 if args.dtype == "f64" else 4

    # ---- inputs: rank 0 builds A; broadcast over NCCL (timed separately) ----
    A = B = None
    if rank == 0 or args.backend == "gloo":
        A, B = load_inputs(args.config, dt)
    t_bcast = None
    if world > 1 and args.backend == "nccl":
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
    seg_local = [r - r0 for r in seg[s0:s1 + 1]]
    plan = acs.Plan(stage_times=True)
    plan.set_segments(seg_local)
    rp_view = dA.row_ptr[r0:r1 + 1]
    nnz_view = int(rp_view[-1].item() - rp_view[0].item())
    view = acs.api._csr_in(dA, row_ptr=rp_view, rows=r1 - r0, nnz=nnz_view)
    stream = torch.cuda.current_stream()

    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    peak = float(peaks.get("hbm_gbs", 6650.0))
    peak_src = "measured" if "hbm_gbs" in peaks else "fallback (B200_PROFILING.md)"

    # warm-up, then the timed region with the clocks sampled during it
    for _ in range(max(args.warmup, 0)):
        C = plan.multiply(dA, dB, stream, A_view=view)
        del C
    torch.cuda.synchronize()
    sampler = ClockSampler(dev.index)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    sampler.start()
    stage_sum = {}
    # N > 1: C stays distributed; each step all-gathers (rows, nnz) per rank for the
    # concatenation offsets
    after = (lambda C: adist.gather_offsets(C.nnz, C.rows, device=cdev)) if world > 1 else None
    ms_total, per_step, st_list = timed_steps(torch, plan, dA, dB, view, stream, args.steps, 0, stage_sum, after)
    clocks = sampler.stop()
    if world > 1:
        dist.barrier()
    info = plan.info()
    ms_step = ms_total / max(args.steps, 1)
    products = info["products"]
    if world > 1:
        tt = torch.tensor([ms_step, statistics.median(per_step), min(per_step)], dtype=torch.float64, device=cdev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms_step_max, med_max, min_max = (float(x) for x in tt.tolist())
        pp = torch.tensor([products, info["nnz_c"]], dtype=torch.int64, device=cdev)
        dist.all_reduce(pp, op=dist.ReduceOp.SUM)
        products_all, nnz_c_all = (int(x) for x in pp.tolist())
    else:
        ms_step_max, med_max, min_max = ms_step, statistics.median(per_step), min(per_step)
        products_all, nnz_c_all = products, info["nnz_c"]
    value = 2.0 * products_all / (ms_step_max * 1e-3) / 1e9

    # ---- method bytes (whole job) and the dominant kernel's roofline (this rank) ----
    mbytes = method_bytes(args.config, vbytes, dA.rows, dA.nnz, dB.rows, dB.nnz, products_all, nnz_c_all)
    method = {"bytes_per_step": mbytes, "GBps": mbytes / (ms_step_max * 1e-3) / 1e9,
              "frac": mbytes / (ms_step_max * 1e-3) / 1e9 / peak,
              "GBps_median_step": mbytes / (med_max * 1e-3) / 1e9,
              "formula": "|A|+|B|[+products*(4+s) if random B]+3*nnz(C)*(4+s)+4*(rows+1) (SURVEY 8(d))"}
    roof = kernel_roofline(args.config, args.dtype, st_list, info, view.rows, nnz_view, dB.rows, dB.nnz, vbytes,
                           peak, peak_src)

    # ---- determinism digests of C (untimed): integer values, then U(-1,1) values ----
    C = plan.multiply(dA, dB, stream, A_view=view)
    dig_int = segment_digest(torch, C, seg_local)
    nnz_c_local = C.nnz
    del C
    vals_u = None
    if rank == 0 or args.backend == "gloo":
        vals_u = np.random.default_rng(2).uniform(-1.0, 1.0, int(dA.nnz)).astype(dt)   # value seed 2
    dU = acs.DeviceCSR(dA.rows, dA.cols, dA.row_ptr, dA.col, torch.empty_like(dA.val))
    if vals_u is not None:
        dU.val.copy_(torch.from_numpy(vals_u))
    if world > 1 and args.backend == "nccl":
        dist.broadcast(dU.val, src=0)
    dUB = dU if args.config != "cfg5" else dB
    planu = acs.Plan()
    planu.set_segments(seg_local)
    viewu = acs.api._csr_in(dU, row_ptr=rp_view, rows=r1 - r0, nnz=nnz_view)
    Cu = planu.multiply(dU, dUB, stream, A_view=viewu)
    dig_u = segment_digest(torch, Cu, seg_local)
    del Cu, dU, dUB
    planu.close()
    torch.cuda.empty_cache()
    if world > 1:
        allv = [None] * world
        dist.all_gather_object(allv, (dig_int, dig_u))
        dig_int = [d for part in allv for d in part[0]]
        dig_u = [d for part in allv for d in part[1]]
    digest = {"int": hashlib.sha256("".join(dig_int).encode()).hexdigest(),
              "uniform": hashlib.sha256("".join(dig_u).encode()).hexdigest(),
              "per_segment": "sha256(row lengths | cols | vals) of each of the 8 canonical segments, "
                             "combined in segment order"}

    # ---- e2e through the public API with host buffers (rank-local) ----
    e2e = None
    if not args.no_e2e:
        e2e = measure_e2e(acs, torch, A, B, dA, dB, view, plan, dev, tdt, rank, world, r0, r1, args, products_all)

    cpu = None
    side = None
    if rank == 0 and world == 1:
        if not args.no_side:
            plan.close()
            torch.cuda.empty_cache()
            side = side_workloads(acs, torch, dev, peak, peak_src, dA2=dA if args.config == "cfg2" else None)
        if not args.no_cpu_baseline:
            try:
                cpu, _ = cpu_oracle_sample(A, B, args.cpu_seconds)
            except Exception as ex:  # never fail the bench line on the baseline
                cpu = {"value": None, "unit": UNIT, "cores": None, "kind": "oracle", "sample": f"failed: {ex}"}

    if rank == 0:
        out = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step_max, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            "config": config_dict(args.config, args.dtype, A, B, products_all) if A is not None else None,
            "ms_per_step_median": med_max, "ms_per_step_min": min_max,
            "method": method,
            "roofline": roof,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": int(info["kernel_launches"]) * args.steps,
            "clocks": clocks,
            "stages_ms_per_step": {k: v / max(args.steps, 1) for k, v in stage_sum.items()},
            "plan": {k: info[k] for k in ("nblocks", "nchunks", "chunk_elems", "nshared", "nmulti", "npath",
                                          "nsearch", "merge_elems", "pool_bytes", "helper_bytes",
                                          "pool_estimate_bytes", "nhash_blocks", "ndict_blocks", "nrow_blocks")},
            "nnz_c": nnz_c_all,
            "parallelism": f"row-segments x{world} ({args.backend})",
            "strategy": "adaptive (hash accumulator per block, per-row accumulator for short rows, AC-ESC "
                        "fallback; DESIGN R31, R34)",
            "side": side,
            "bcast_s": t_bcast,
            "digest": digest,
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
        tt = torch.tensor([ms], dtype=torch.float64, device=dev if dist.get_backend() == "nccl" else "cpu")
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
