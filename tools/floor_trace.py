"""Kernel timeline of one rank's share (the per-multiply fixed floor).

Multiplies the share of rank g of N (canonical 8 segments) a few times and records the
last multiply with torch.profiler (CUPTI): every kernel / memcpy / memset with its start,
duration and the idle gap before it, so the non-scaling part of a multiply (launch and
read-back latency, tiny kernels) can be read off directly.

usage: python tools/floor_trace.py [cfg2] [N=8] [g=0] [f64|f32]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from torch.profiler import ProfilerActivity, profile

import paper_conf_ppopp_wintermzss19_b200 as acs
from paper_conf_ppopp_wintermzss19_b200 import dist as adist
from synth import config

cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg2"
N = int(sys.argv[2]) if len(sys.argv) > 2 else 8
g = int(sys.argv[3]) if len(sys.argv) > 3 else 0
dt = np.float32 if len(sys.argv) > 4 and sys.argv[4] == "f32" else np.float64
A, B = config(cfg, dt)
dA = acs.DeviceCSR.from_host(A, "cuda", dt)
dB = dA if cfg != "cfg5" else acs.DeviceCSR.from_host(B, "cuda", dt)
seg = acs.canonical_segments(dA, 8)
stream = torch.cuda.current_stream()
s0, s1 = adist.rank_segments(8, N, g)
plan = acs.Plan()
r0, r1 = seg[s0], seg[s1]
plan.set_segments(adist.local_segment_rows(seg, s0, s1))
rp = dA.row_ptr[r0:r1 + 1]
view = acs.api._csr_in(dA, row_ptr=rp, rows=r1 - r0, nnz=int(rp[-1].item() - rp[0].item()))
for _ in range(5):
    C = plan.multiply(dA, dB, stream, A_view=view)
    del C
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
    e0.record(stream)
    C = plan.multiply(dA, dB, stream, A_view=view)
    e1.record(stream)
    torch.cuda.synchronize()
# host-side split of one multiply (no profiler): symbolic (ends with the nnz read-back),
# C allocation, numeric launches
import time
hs = []
for _ in range(5):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    nnz = plan.symbolic(dA, dB, stream, view)
    t1 = time.perf_counter()
    rp_ = torch.empty(plan._rows + 1, dtype=torch.int32, device="cuda")
    col_ = torch.empty(max(nnz, 1), dtype=torch.int32, device="cuda")
    val_ = torch.empty(max(nnz, 1), dtype=dA.dtype, device="cuda")
    t2 = time.perf_counter()
    plan.numeric(rp_, col_, val_, stream)
    t3 = time.perf_counter()
    torch.cuda.synchronize()
    t4 = time.perf_counter()
    hs.append((t1 - t0, t2 - t1, t3 - t2, t4 - t3))
    del rp_, col_, val_
hs = [sorted(x)[len(x) // 2] * 1e6 for x in zip(*hs)]
print("host us (median): symbolic %.1f  alloc %.1f  numeric-launch %.1f  numeric-drain %.1f" % tuple(hs))
ev = [e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA]
ev.sort(key=lambda e: e.time_range.start)
rows, prev_end, t0 = [], None, ev[0].time_range.start if ev else 0
for e in ev:
    st, en = e.time_range.start, e.time_range.end
    rows.append({"name": e.name[:60], "start_us": round(st - t0, 1), "dur_us": round(en - st, 1),
                 "gap_us": round(st - prev_end, 1) if prev_end is not None else 0.0})
    prev_end = max(prev_end or en, en)
busy = sum(r["dur_us"] for r in rows)
span = (prev_end - t0) if ev else 0
for r in rows:
    print(f'{r["start_us"]:9.1f} {r["dur_us"]:8.1f} gap {r["gap_us"]:7.1f}  {r["name"]}')
print(json.dumps({"workload": cfg, "N": N, "rank": g, "events": len(rows), "span_us": round(span, 1),
                  "busy_us": round(busy, 1), "idle_us": round(span - busy, 1),
                  "event_ms": round(e0.elapsed_time(e1), 4)}))
