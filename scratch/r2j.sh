cd $GRAFT_REPO_ROOT
timeout 240 python -m pytest tests/test_gpu_hash.py tests/test_gpu_spa.py tests/test_gpu_dict.py -q -x 2>&1 | tail -3
timeout 120 python tools/strat_cmp.py cfg2 f64 hash,adaptive 2>&1 | tail -3
timeout 120 python tools/strat_cmp.py cfg2 f32 hash 2>&1 | tail -2
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_hash -s 1 -c 1 -o gpurun_out/r2j_hash_cfg2_f64 python scratch/one.py cfg2 f64 hash > gpurun_out/r2j_p1.log 2>&1
