mkdir -p gpurun_out; rm -f gpurun_out/var.txt
L=paper_conf_ppopp_wintermzss19_b200
for v in "" _prev; do
  ACSPGEMM_LIB=$PWD/$L/libacspgemm$v.so python -m pytest tests/test_gpu_hash.py -q -k "stale or reuse" > gpurun_out/stale$v.log 2>&1
  for dt in f64 f32; do
    ACSPGEMM_LIB=$PWD/$L/libacspgemm$v.so python tools/strat_cmp.py cfg2 $dt adaptive 10 2>&1 | head -1 | sed "s/^/var$v /" >> gpurun_out/var.txt
  done
done
