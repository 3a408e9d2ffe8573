import sys, os
sys.path.insert(0, sys.argv[1]); sys.path.insert(1, os.getcwd()); sys.path.insert(2, os.path.join(os.getcwd(), "tests"))
import numpy as np
import paper_conf_ppopp_wintermzss19_b200 as p
print(p.SO_PATH)
from oracle import alg
ok = True
for seed in range(20):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 2049)); rows = rng.integers(0, int(rng.choice([1,3,40,500])), n).astype(np.int32)
    cols = rng.integers(0, int(rng.choice([1,5,100,70000,3000000])), n).astype(np.int32)
    vals = rng.integers(-9, 10, n).astype(np.float64)
    orow, ocol, oval, ost = p.debug_sort_compact(rows, cols, vals)
    order = np.lexsort((np.arange(n), cols, rows))
    ok &= bool((orow == rows[order]).all() and (ocol == cols[order]).all())
print("sort ok", ok)
