"""multiply (symbolic + numeric, host syncs) vs numeric_update (graph replay, no syncs)."""
import sys, os, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import config
st = torch.cuda.Stream()
for cfg in sys.argv[1].split(",") if len(sys.argv) > 1 else ["cfg1", "cfg2"]:
    A, B = config(cfg)
    with torch.cuda.stream(st):
        dA = acs.DeviceCSR.from_host(A, "cuda"); dB = dA if cfg != "cfg5" else acs.DeviceCSR.from_host(B, "cuda")
        plan = acs.Plan()
        C = plan.multiply(dA, dB, st)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = 50 if cfg == "cfg1" else 10
        for _ in range(3): C2 = plan.multiply(dA, dB, st); del C2
        st.synchronize(); e0.record(st)
        for _ in range(reps): C2 = plan.multiply(dA, dB, st); del C2
        e1.record(st); st.synchronize(); t_mult = e0.elapsed_time(e1) / reps
        C = plan.multiply(dA, dB, st)
        for _ in range(3): plan.numeric_update(dA, dB, C, st)
        st.synchronize(); e0.record(st)
        for _ in range(reps): plan.numeric_update(dA, dB, C, st)
        e1.record(st); st.synchronize(); t_upd = e0.elapsed_time(e1) / reps
        print(json.dumps({"workload": cfg, "multiply_ms": t_mult, "numeric_update_ms": t_upd}), flush=True)
        plan.close()
