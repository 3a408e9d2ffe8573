#!/bin/bash
for lib in paper_conf_ppopp_wintermzss19_b200/libacspgemm*.so; do
  ACSPGEMM_LIB=$PWD/$lib python scratch/strat.py f64 128 hash 2>&1 | cut -c1-140
  ACSPGEMM_LIB=$PWD/$lib python scratch/strat.py f32 128 hash 2>&1 | cut -c1-140
done
