"""No dead knobs (CPU, no GPU): two settings of the space that differ in one field must
generate different sm_100a code (SASS via cuobjdump) or a different launch geometry.

For one base setting per kernel path, every valid one-step neighbour in every field
(Table I, plus bt / qstore) is compiled through cst_variant_cubin and compared
with the base (tools/knob_audit.py).  Round 1 shipped UF_x / UF_y on the fast streaming
paths, every UF on the TMEM paths, prefetch without staging and rhs4's use_retiming as
no-ops; the space rules R6 / R9 / R16 now pin those fields to their canonical value, and
this test keeps it that way.  The full audit (22 bases, 363 pairs) is
`python tools/knob_audit.py`."""
import importlib.util
import os
import shutil
import tempfile

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SUBSET = {"star4_tma_ret", "star4_ldst", "star4_tmem", "star4_generic", "star4_tile3d",
          "star1_tblock", "hyp_tmem", "hyp_reg", "rhs4_bmz2", "box_l1", "rhs4_ret"}


@pytest.mark.skipif(shutil.which("cuobjdump") is None, reason="cuobjdump not found")
def test_one_step_neighbours_generate_distinct_code():
    spec = importlib.util.spec_from_file_location("knob_audit",
                                                  os.path.join(ROOT, "tools", "knob_audit.py"))
    A = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(A)
    bases = [b for b in A.BASES if b[0] in SUBSET]
    assert len(bases) == len(SUBSET)
    with tempfile.TemporaryDirectory() as td:
        dead, checked = A.audit(bases, 64, os.cpu_count() or 4, td)
    assert checked >= 120, checked
    assert dead == [], dead
