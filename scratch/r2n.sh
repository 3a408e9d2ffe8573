cd $GRAFT_REPO_ROOT
timeout 400 python -m pytest tests/test_gpu_parity.py -q -x -k "long_row_chunks or long_rows or dense_row or giant or bit_identical or path_merge" 2>&1 | tail -3
timeout 600 python -m pytest tests/test_gpu_fullsize.py -q -x -k "graph500 or cfg3_rmat_full and float64" 2>&1 | tail -3
timeout 300 python -m pytest tests/test_gpu_dist.py -q -x 2>&1 | tail -3
timeout 900 python tools/scaling_proxy.py cfg2 > gpurun_out/r2n_scaling_cfg2.json 2>&1; tail -c 1500 gpurun_out/r2n_scaling_cfg2.json
