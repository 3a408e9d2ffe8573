cd $GRAFT_REPO_ROOT
cat > /tmp/t.py <<'PY'
import sys, os
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.getcwd() + "/tests")
import numpy as np
from test_gpu_dict import banded_b, run, window_a
rng = np.random.default_rng(9)
nb = 3000
B = banded_b(nb, 16 * nb + 64, 16, 32, rng)
A = window_a(2000, nb, 8, rng)
out, info = run(A, B, np.float64, strategy="adaptive")
print({k: info[k] for k in ("nblocks", "nspa_blocks", "nhash_blocks")})
PY
ACSPGEMM_LIB=$PWD/paper_conf_ppopp_wintermzss19_b200/libacspgemm_dbg.so python /tmp/t.py 2>&1 | tail -30
