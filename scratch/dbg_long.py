import sys; sys.path.insert(0,'.')
import numpy as np, torch
sys.path.insert(0, "tests"); from test_gpu_parity import *
A = power_law_csr(3000, 3000, mean_len=12, alpha=1.2, max_len=1500, seed=0)
B = power_law_csr(3000, 3000, mean_len=12, alpha=1.2, max_len=3000, seed=10)
print("products", oracle.products(A,B), "nnzA", A.nnz)
plan = pkg().Plan()
try:
    assert_parity(A, B, np.float64, plan=plan)
    print("OK", plan.info())
except Exception as e:
    print("FAIL", e)
