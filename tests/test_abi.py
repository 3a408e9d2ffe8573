"""CPU checks of the boundary: the C-ABI library builds, loads and exports every symbol
include/acspgemm.h declares; host-only entry points behave (no GPU compute calls)."""
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    src = open(os.path.join(ROOT, "include", "acspgemm.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(acspgemm_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_header_symbol():
    import paper_conf_ppopp_wintermzss19_b200 as pkg
    lib = pkg.load()
    names = header_functions()
    assert len(names) >= 18
    for n in names:
        assert hasattr(lib, n), n
    # the binding declares a signature for each of them
    assert set(names) == set(pkg.SIGNATURES)


def test_host_only_entry_points():
    import paper_conf_ppopp_wintermzss19_b200 as pkg
    lib = pkg.load()
    assert lib.acspgemm_abi_version() == 2
    assert pkg.const("NPB") == 512 and pkg.const("CAP") == 2048 and pkg.const("KEEP") == 4 * pkg.const("THREADS")
    assert lib.acspgemm_const(99) == -1
    assert lib.acspgemm_status_string(0) == b"ok"
    assert lib.acspgemm_status_string(2) == b"dimension mismatch"


def test_pool_estimate_matches_oracle():
    """K10 in the library vs the oracle's step-by-step formula."""
    import paper_conf_ppopp_wintermzss19_b200 as pkg
    from oracle import alg
    cases = [(13514, 352762, 13514, 13514, 352762, 8), (29089, 2852184, 957432, 29089, 2852184, 8),
             (1489752, 10319760, 1489752, 1489752, 10319760, 4), (10, 20, 40, 40, 1600, 8), (0, 0, 1, 1, 0, 8)]
    for c in cases:
        assert pkg.pool_estimate_bytes(*c) == pytest.approx(alg.pool_estimate_bytes(*c), rel=1e-12)


def test_no_oracle_import_in_product():
    """The product path never imports the oracle (and vice versa)."""
    pkgdir = os.path.join(ROOT, "paper_conf_ppopp_wintermzss19_b200")
    for dirpath, _, files in os.walk(pkgdir):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c")):
            txt = open(os.path.join(ROOT, "oracle", f)).read()
            assert "import paper_conf_ppopp_wintermzss19_b200" not in txt, f
            assert "from paper_conf_ppopp_wintermzss19_b200" not in txt, f


def test_binding_fails_loudly_without_library(tmp_path, monkeypatch):
    import paper_conf_ppopp_wintermzss19_b200._lib as L
    monkeypatch.setattr(L, "SO_PATH", str(tmp_path / "missing.so"))
    monkeypatch.setattr(L, "_lib", None)
    with pytest.raises(ImportError):
        L.load()
