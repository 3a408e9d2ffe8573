cd $GRAFT_REPO_ROOT
for lib in libacspgemm.so libacspgemm_cpa.so; do
  for c in cfg3 cfg5; do
    ACSPGEMM_LIB=$PWD/paper_conf_ppopp_wintermzss19_b200/$lib timeout 300 python tools/strat_cmp.py $c f64 adaptive 5 2>&1 | head -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$lib', '$c', round(d['ms'],2), 'ESC', d['stages']['ESC'], d['sha'])"
  done
  ACSPGEMM_LIB=$PWD/paper_conf_ppopp_wintermzss19_b200/$lib timeout 300 python tools/strat_cmp.py cfg2 f64 esc 5 2>&1 | head -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$lib', 'cfg2-esc', round(d['ms'],2), 'ESC', d['stages']['ESC'], d['sha'])"
done
ACSPGEMM_LIB=$PWD/paper_conf_ppopp_wintermzss19_b200/libacspgemm_cpa.so timeout 600 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k "regex:acs::k_esc<" -s 1 -c 1 -o gpurun_out/r2s_esc_cpa_cfg5_f64 python scratch/one.py cfg5 f64 > gpurun_out/r2s_p1.log 2>&1
