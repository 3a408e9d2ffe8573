cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x --deselect tests/test_gpu_fullsize.py 2>&1 | tail -2
timeout 900 python tools/scaling_proxy.py cfg2 > gpurun_out/r2r_scaling_cfg2.json 2>&1; python -c "
import json; d=json.load(open('gpurun_out/r2r_scaling_cfg2.json'))
for n,r in d['results'].items(): print(n, round(r['T_ms'],3), round(r['efficiency'],3), r['slowest_rank_stages_ms'])"
