"""CPU oracle for recursive classical Gram-Schmidt QR -- TEST INFRASTRUCTURE ONLY.

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s `cpu_baseline` /
`--impl reference` legs may import or execute anything under `oracle/`.  The
product path (`paper_conf_icpp_zhangw21_b200/`, `include/`, the CUDA library)
never imports it and shares no code with it; the only common dependency is the
seeded input generators in `rgsqr_inputs/`, which hold none of the method's
arithmetic.

Contents (each function cites the PAPER.md passage it follows):

* ``cgs.py``    -- O1 column CGS (Eq. 1), O2 CGS2, O3 recursive CGS (Eq. 2),
                   O4 blocked CGS (section 3.1.2), O5 precision-emulating recursive CGS,
                   O6 recursive CGS2 (reorthogonalized).
* ``checks.py`` -- backward error, orthogonality loss, triangularity, R error,
                   Gram-Cholesky reference R for large inputs.
* ``model.py``  -- recursion shapes, flop count, the paper's data-movement models.

Pins (tests/test_oracle_*.py, `-m "not gpu"`): Householder QR with sign
normalisation, Cholesky of X^T X, closed forms for n <= 2, Hadamard (R = I),
diagonal scaling (R = D), exact dyadic mixing (R = R0), invariants, and the
paper's printed shape / byte formulas (tests/golden/).  O5 is pinned two-sided
(tests/test_oracle_emulation_pins.py): the closed-form backward error of RN storage
rounding, 0.4247 u sqrt(1 + L/2), and the independent emulation table of SURVEY.md:618-626.
The executor-shaped byte splits of model.py are tied to PAPER.md:141/145 and to the
reading-R11 count by exact identities (tests/test_model_pins.py).  Parity status per
function: DESIGN.md section 4.
"""
from .cgs import cgs, cgs2, rgs, rgs2, blocked_cgs, rgs_emulated, QRResult  # noqa: F401
from .checks import (backward_error, orthogonality, r_rel_error, is_upper_triangular,  # noqa: F401
                     gram_cholesky_r)
from . import model  # noqa: F401
