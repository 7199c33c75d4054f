"""The C-ABI boundary: libsomier.so loads and exports every symbol that
include/*.h declares, with no torch types involved. No compute calls here."""
import ctypes
import os
import re
import subprocess

import pytest

import paper_conf_ipps_torresft22_b200 as P
from paper_conf_ipps_torresft22_b200 import _native as N

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    names = []
    for h in ("spread.h", "somier.h"):
        text = open(os.path.join(ROOT, "include", h)).read()
        text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
        names += re.findall(r"^\s*(?:const\s+)?[a-z_]+[\s\*]+((?:spread|somier)_[a-z0-9_]+)\s*\(", text, re.M)
    return sorted(set(names))


def test_every_declared_symbol_is_exported_and_bound():
    L = N.lib()
    declared = _declared()
    assert len(declared) >= 25
    for name in declared:
        assert hasattr(L, name), name
    bound = {s[0] for s in N.SIGNATURES}
    assert set(declared) == bound


def test_exports_match_nm():
    out = subprocess.run(["nm", "-D", "--defined-only", N.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T ((?:spread|somier)_\w+)", out))
    assert set(_declared()) <= exported


def test_library_links_no_torch():
    out = subprocess.run(["ldd", N.LIB_PATH], capture_output=True, text=True).stdout
    assert "torch" not in out and "c10" not in out
    out = subprocess.run(["cuobjdump", "--list-elf", N.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_status_strings_and_version():
    assert N.status_string(0) == "SPREAD_OK"
    assert N.status_string(-7) == "SPREAD_ESTATE"
    assert "sm_100a" in P.version()


def test_struct_layouts():
    # include/somier.h: somier_params = 3*8 + 7*8 + 4*4 bytes; somier_stats_t = 16*8
    assert ctypes.sizeof(N.somier_params) == 96
    assert ctypes.sizeof(N.somier_stats_t) == 8 * (1 + 3 + 1 + 3 + 3 + 1 + 1)


def test_stats_combine_is_exact_host_logic():
    """somier_stats_combine is host arithmetic: int128 sums add exactly."""
    sp = P.SomierParams(n=(4, 4, 4))
    big = (1 << 100) + 12345
    a = P.Stats(3, (0.0,) * 3, 0.0, (big, -big, 7), 0x3FF0000000000000, 32)
    b = P.Stats(3, (0.0,) * 3, 0.0, (-(1 << 100), big, -7), 0x4000000000000000, 32)
    c = P.combine_stats([a, b], sp)
    assert c.sums == (12345, 0, 0)
    assert c.vmax == 2.0 ** 0.5 and c.nodes == 64
    assert c.centre[0] == (12345 * 2.0 ** -60) / 64
    with pytest.raises(P.SpreadError):
        P.combine_stats([a, P.Stats(4, (0.0,) * 3, 0.0, (0, 0, 0), 0, 0)], sp)


def test_stats_combine_propagates_out_of_domain():
    """A partial outside the exact-stats domain (NaN centre, include/somier.h)
    makes the combined centre NaN; the sums and vmax still combine exactly."""
    import math

    sp = P.SomierParams(n=(4, 4, 4))
    a = P.Stats(3, (1.0, 2.0, 3.0), 0.0, (5, 6, 7), 0x3FF0000000000000, 32)
    b = P.Stats(3, (math.nan,) * 3, 0.0, (1, 1, 1), 0x4000000000000000, 32)
    c = P.combine_stats([a, b], sp)
    assert not c.in_domain and all(math.isnan(x) for x in c.centre)
    assert c.sums == (6, 7, 8) and c.vmax == 2.0 ** 0.5
    d = P.combine_stats([a, a], sp)
    assert d.in_domain and d.centre[0] == (10 * 2.0 ** -60) / 64


def test_somier_init_without_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(P.SpreadError) as e:
        P.Somier(P.Spread([0], 1, 8), P.SomierParams(n=(10, 10, 10)))
    assert e.value.status == N.ENODEV


def test_capi_exposes_every_entry_point_under_its_c_name():
    """The Python binding carries the C names (argument marshalling only)."""
    from paper_conf_ipps_torresft22_b200 import capi

    for name in _declared():
        assert callable(getattr(capi, name)), name
    # host-only calls work without a GPU, through the C names
    h = ctypes.c_void_p()
    devs = (ctypes.c_int * 3)(2, 0, 1)
    capi.spread_create(devs, 3, 1, 14, 0, 4, ctypes.byref(h))
    n = ctypes.c_int64()
    capi.spread_num_chunks(h, ctypes.byref(n))
    assert n.value == 4  # range of 14 iterations in chunks of 4: 4, 4, 4, 2
    capi.spread_destroy(h)
    with pytest.raises(P.SpreadError):
        capi.spread_create(devs, 0, 1, 14, 0, 4, ctypes.byref(h))  # no devices
    assert capi.somier_version()


def test_host_grid_size_is_checked():
    """The binding refuses a host grid whose element count differs from what
    the C side reads or writes (n0*n1*n2 per grid) instead of letting C run off
    its end."""
    import numpy as np
    import pytest as _pytest

    from paper_conf_ipps_torresft22_b200 import somier as S

    ok = np.zeros(24)
    assert S._dptr(ok, 24) is not None
    with _pytest.raises(ValueError):
        S._dptr(np.zeros(23), 24)
    with _pytest.raises(TypeError):
        S._dptr(np.zeros(24, dtype=np.float32), 24)


def test_struct_layouts_match_the_c_header(tmp_path):
    """The ctypes mirrors have the C compiler's sizes and field offsets."""
    import shutil
    import subprocess

    cc = shutil.which("gcc") or shutil.which("cc")
    if cc is None:
        pytest.skip("no C compiler")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    structs = {"somier_params": N.somier_params, "somier_stats_t": N.somier_stats_t}
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "somier.h"', "int main(void) {"]
    for name, ct in structs.items():
        lines.append('printf("%s %%zu\\n", sizeof(%s));' % (name, name))
        for f in ct._fields_:
            lines.append('printf("%s.%s %%zu\\n", offsetof(%s, %s));' % (name, f[0], name, f[0]))
    lines.append("return 0; }")
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines) + "\n")
    exe = tmp_path / "layout"
    subprocess.run([cc, "-std=c99", "-I", os.path.join(root, "include"), str(src), "-o", str(exe)], check=True)
    out = dict(l.rsplit(" ", 1) for l in subprocess.run([str(exe)], check=True, capture_output=True,
                                                         text=True).stdout.splitlines())
    for name, ct in structs.items():
        assert int(out[name]) == ctypes.sizeof(ct), name
        for f in ct._fields_:
            assert int(out["%s.%s" % (name, f[0])]) == getattr(ct, f[0]).offset, (name, f[0])
