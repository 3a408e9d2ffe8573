cd $GRAFT_REPO_ROOT
for t in su4 su8 su16 su16w8 su32; do
  ACSPGEMM_LIB=$PWD/paper_conf_ppopp_wintermzss19_b200/libacspgemm_$t.so timeout 300 python tools/strat_cmp.py cfg2 f64 adaptive 5 2>&1 | head -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$t', d['ms'], d['stages']['DICT'], d['sha'])"
done
