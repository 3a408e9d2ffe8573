cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_spa.py tests/test_gpu_dict.py tests/test_gpu_hash.py -x -q 2>&1 | tail -15
timeout 300 python tools/strat_cmp.py cfg2 f64 adaptive,hash,dict 2>&1 | tail -5
timeout 300 python tools/strat_cmp.py cfg2 f32 adaptive,hash,dict 2>&1 | tail -5
