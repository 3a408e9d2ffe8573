#!/bin/bash
for lib in paper_conf_ppopp_wintermzss19_b200/libacspgemm*.so; do
  echo $lib; ACSPGEMM_LIB=$PWD/$lib python scratch/allcfg.py cfg3,cfg5 2>&1 | python3 -c "
import sys, json
for l in sys.stdin:
    try: d=json.loads(l)
    except: continue
    print(d['workload'], d['dtype'], round(d['ms_per_multiply'],2), {k: round(d['stages_ms'][k],2) for k in ('ESC','MM','PM','CC')})
"
done
