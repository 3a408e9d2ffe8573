#!/bin/bash
# all built variants x dtypes (GPU box)
for lib in paper_conf_ppopp_wintermzss19_b200/libacspgemm*.so; do
  for dt in f64 f32; do ACSPGEMM_LIB=$PWD/$lib python scratch/strat.py $dt; done
done
