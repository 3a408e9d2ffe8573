cd $GRAFT_REPO_ROOT
for t in w3 w6 w8; do
  ACSPGEMM_LIB=$PWD/paper_conf_ppopp_wintermzss19_b200/libacspgemm_$t.so timeout 120 python tools/strat_cmp.py cfg2 f64 hash 5 2>&1 | head -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$t', d['ms'], d['stages']['HASH'], d['sha'])"
done
