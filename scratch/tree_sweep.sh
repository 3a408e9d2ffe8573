for M in 0 2 3 4 8; do
  ACS_EXTRA_NVCC_FLAGS="-DACS_TREE_MAX_M=$M" python -c "from paper_conf_ppopp_wintermzss19_b200 import build; build.build(force=True)" >/dev/null 2>&1
  echo "M=$M"; python scratch/allcfg.py cfg3,cfg5 | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print(d['workload'], d['dtype'], round(d['ms_per_multiply'],2), d['stages_ms']['PM'], d['stages_ms']['MM'])"
done
