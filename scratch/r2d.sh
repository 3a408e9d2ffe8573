cd $GRAFT_REPO_ROOT
ACSPGEMM_LIB=$PWD/paper_conf_ppopp_wintermzss19_b200/libacspgemm_dbg.so timeout 300 python -m pytest tests/test_gpu_spa.py -x -q -k "halving and float64" 2>&1 | grep "spa fail" | head -40
timeout 600 python -m pytest tests/test_gpu_spa.py -q 2>&1 | tail -4
timeout 300 python tools/strat_cmp.py cfg2 f64 adaptive,hash 2>&1 | tail -3
ncu --set full --import-source on --clock-control none -k regex:k_spa -s 1 -c 1 -o gpurun_out/r2d_spa_cfg2_f64 python scratch/one.py cfg2 f64 > gpurun_out/r2d_p1.log 2>&1
