cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_spa.py -q 2>&1 | tail -3
timeout 300 python tools/strat_cmp.py cfg2 f64 adaptive,hash 2>&1 | tail -3
ncu --set full --import-source on --clock-control none -k regex:k_spa -s 1 -c 1 -o gpurun_out/r2f_spa_cfg2_f64 python scratch/one.py cfg2 f64 > gpurun_out/r2f_p1.log 2>&1
