"""Seeded synthetic input generators (shared by oracle tests, GPU tests, bench).
Holds no SpGEMM arithmetic."""
from .matrices import (CSR, from_coo, transpose, poisson2d_5pt, poisson3d_27pt, poisson3d_7pt,
                       aggregation_prolongator, rmat, lp_like, random_csr, random_rowlen_csr,
                       power_law_csr, config)

__all__ = ["CSR", "from_coo", "transpose", "poisson2d_5pt", "poisson3d_27pt", "poisson3d_7pt",
           "aggregation_prolongator", "rmat", "lp_like", "random_csr", "random_rowlen_csr",
           "power_law_csr", "config"]
