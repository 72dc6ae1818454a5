"""CPU-side checks of the boundary: the shared library builds, loads and exports every
symbol include/rgsqr.h declares (no compute calls without a GPU)."""
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "rgsqr.h")).read()
    return sorted(set(re.findall(r"\b(rgsqr_[a-z_]+)\s*\(", src)))


def test_header_lists_north_star_calls():
    d = _declared()
    for name in ("rgsqr_create", "rgsqr_factor", "rgsqr_destroy"):
        assert name in d


def test_library_exports_all_declared_symbols():
    from paper_conf_icpp_zhangw21_b200 import build, rgsqr
    lib = build.build()
    out = subprocess.run(["nm", "-D", "--defined-only", lib], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\s[TW]\s(rgsqr_\w+)", out))
    missing = [s for s in _declared() if s not in exported]
    assert not missing, missing
    assert sorted(rgsqr.EXPORTS) == sorted(_declared())
    L = rgsqr.load_library()
    assert L.rgsqr_version() == 100
    assert L.rgsqr_status_string(-2) == b"RGSQR_ERR_BUDGET_TOO_SMALL"


def test_create_fails_cleanly_without_gpu():
    import torch
    if torch.cuda.is_available():
        return
    from paper_conf_icpp_zhangw21_b200 import Handle, RgsqrError
    try:
        Handle(0)
    except RgsqrError as e:
        assert e.status < 0
    else:
        raise AssertionError("create must fail without a device")
