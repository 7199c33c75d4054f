"""The pins catch the two mistakes round 1's pins let through (VERDICT r01:
a = F*M instead of F/M, and the spring rest length read from the lattice
spacing): each mutant of oracle/somier_oracle.c is compiled and the pins that
target it -- C2 at M != 1 and C8 on a pre-stressed chain -- must fail.
tools/mutate_oracle.py runs the whole pin suite against 22 mutants
(profiles/r02_oracle_mutants.json)."""
import os
import shutil
import sys
import tempfile

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))

import mutate_oracle as M  # noqa: E402

pytestmark = pytest.mark.skipif(shutil.which("gcc") is None, reason="needs gcc")


@pytest.mark.parametrize("name,select", [("accel_f_times_m", "two_mass or chain"),
                                         ("forces_rest_len_is_spacing", "chain")])
def test_targeted_pins_kill_mutant(name, select):
    base = open(M.SRC).read()
    orig, mut = {n: (o, m) for n, o, m in M.MUTANTS}[name]
    assert base.count(orig) == 1
    with tempfile.TemporaryDirectory() as td:
        lib = os.path.join(td, "m.so")
        M.build(base.replace(orig, mut), lib)
        rc, failed, _ = M.run_pins(lib, select=select, timeout=300)
        assert rc != 0 and failed, "mutant %s survived the %r pins" % (name, select)
        lib0 = os.path.join(td, "o.so")
        M.build(base, lib0)
        rc0, failed0, _ = M.run_pins(lib0, select=select, timeout=300)
        assert rc0 == 0, failed0
