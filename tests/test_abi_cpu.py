"""CPU-side checks of the C-ABI library: it builds, loads, exports every
symbol include/mas_pcg.h declares, and rejects bad meshes before touching a
device (no compute calls: there is no GPU here)."""
import math
import os
import re

import numpy as np
import pytest

from paper_conf_ipps_caplansl23_b200 import build as B
from paper_conf_ipps_caplansl23_b200 import workloads as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def mp():
    B.build()
    from paper_conf_ipps_caplansl23_b200 import maspcg
    return maspcg


def header_symbols():
    src = open(os.path.join(ROOT, "include", "mas_pcg.h")).read()
    return set(re.findall(r"^MAS_API[^(]*?\b(mas_\w+)\s*\(", src, flags=re.M))


def test_exports_every_declared_symbol(mp):
    declared = header_symbols()
    assert len(declared) >= 14
    assert declared == set(mp.ABI_SYMBOLS)
    import ctypes
    L = ctypes.CDLL(B.SO)
    for name in declared:
        assert hasattr(L, name), name


def test_sass_is_sm100a():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", B.build()],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_version_and_status_strings(mp):
    assert "sm_100a" in mp.mas_version()
    for s in range(7):
        assert mp.status_string(s)
    assert mp.status_string(99) == "unknown status"


def mesh_args(m):
    return [m.rF, m.rC, m.tF, m.tC, m.pF, m.pC]


@pytest.mark.parametrize("mutate,frag", [
    (lambda a: a[0].__setitem__(3, a[0][2]), "r_node is not strictly increasing"),
    (lambda a: a[1].__setitem__(0, a[0][0]), "r_half[0] is not inside"),
    (lambda a: a[4].__setitem__(-1, a[4][-1] * 0.99), "2 pi"),
    (lambda a: a[2].__setitem__(0, 0.01), "north pole"),
    (lambda a: a[2].__setitem__(-1, math.pi - 1e-6), "south pole"),
])
def test_grid_validation_errors(mp, mutate, frag):
    m = W.stretched_mesh(4, 6, 8)
    args = [np.array(a) for a in mesh_args(m)]
    mutate(args)
    with pytest.raises(mp.MasError) as e:
        mp.mas_grid_create(*args, pole_flags=3)
    assert e.value.status == mp.MAS_ERR_ARG
    assert frag in mp.last_error()


def test_grid_validation_odd_np_and_ranks(mp):
    m = W.stretched_mesh(4, 6, 9)
    with pytest.raises(mp.MasError) as e:
        mp.mas_grid_create(*mesh_args(m))
    assert "even" in mp.last_error()
    m = W.stretched_mesh(2, 6, 8)
    with pytest.raises(mp.MasError):
        mp.mas_grid_create(*mesh_args(m), dist=(4, 0, bytes(128)))
    assert "nranks" in mp.last_error()


def test_no_device_is_a_loud_error(mp):
    """A valid mesh on a box without a GPU fails with MAS_ERR_CUDA (no CPU
    fallback exists)."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    m = W.stretched_mesh(4, 6, 8)
    with pytest.raises(mp.MasError) as e:
        mp.mas_grid_create(*mesh_args(m))
    assert e.value.status == mp.MAS_ERR_CUDA


def test_product_package_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_caplansl23_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
                src = open(os.path.join(dirpath, f)).read()
                assert "mas_ref" not in src and "import oracle" not in src \
                    and "from oracle" not in src, f
