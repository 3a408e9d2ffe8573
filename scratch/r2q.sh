cd $GRAFT_REPO_ROOT
timeout 400 python -m pytest tests/test_gpu_hash.py tests/test_gpu_dict.py tests/test_gpu_parity.py -q -x 2>&1 | tail -2
timeout 120 python tools/strat_cmp.py cfg2 f64 adaptive 2>&1 | tail -2
timeout 900 python tools/scaling_proxy.py cfg2 > gpurun_out/r2q_scaling_cfg2.json 2>&1; python -c "
import json; d=json.load(open('gpurun_out/r2q_scaling_cfg2.json'))
for n,r in d['results'].items(): print(n, round(r['T_ms'],3), round(r['efficiency'],3), r['slowest_rank_stages_ms'])"
