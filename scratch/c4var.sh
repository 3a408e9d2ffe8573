#!/bin/bash
for lib in paper_conf_ppopp_wintermzss19_b200/libacspgemm*.so; do echo $lib; ACSPGEMM_LIB=$PWD/$lib python scratch/cfg4info.py 2>&1 | cut -c1-120; done
