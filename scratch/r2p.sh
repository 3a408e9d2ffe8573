cd $GRAFT_REPO_ROOT
timeout 400 python -m pytest tests/test_gpu_parity.py tests/test_gpu_hash.py tests/test_gpu_budget.py tests/test_gpu_update.py -q -x 2>&1 | tail -2
timeout 600 python -m pytest tests/test_gpu_fullsize.py -q -x -k "graph500 or cfg3_rmat_full" 2>&1 | tail -2
timeout 300 python tools/g500_time.py 18 3
ACSPGEMM_LIB=$PWD/paper_conf_ppopp_wintermzss19_b200/libacspgemm_noptr.so timeout 300 python tools/g500_time.py 18 3
timeout 600 python tools/g500_time.py 20 2
ACSPGEMM_LIB=$PWD/paper_conf_ppopp_wintermzss19_b200/libacspgemm_noptr.so timeout 600 python tools/g500_time.py 20 2
