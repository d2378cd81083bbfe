"""CPU checks of bench.py's reported-figure helpers.

The algorithmic bytes per cell that the roofline objects divide by are
checked against what the hardware measured, not retyped: the committed ncu
captures (profiles/ncu_*.json, dram__bytes_read + dram__bytes_write of one
launch) divided by the cells of that launch must land within a few percent
of bench.py's per-cell figure (DRAM traffic can only exceed the algorithmic
minimum by re-reads, or undercut it by L2 hits).  The config shapes are
parsed from BASELINE.json's own config strings."""
import importlib.util
import json
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def load_bench():
    spec = importlib.util.spec_from_file_location("bench", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


@pytest.mark.parametrize("prof,which", [
    ("ncu_C3_kernelA.json", "A"),
    ("ncu_C3_kernelB.json", "B"),
    ("ncu_C2a_kaniso.json", "Lpar"),
])
def test_algorithmic_bytes_match_measured_dram_traffic(prof, which):
    b = load_bench()
    path = os.path.join(ROOT, "profiles", prof)
    d = json.load(open(path))
    cfg = "C3" if "C3" in prof else "C2a"
    kind, nr, nt, np_ = b.CONFIGS[cfg]
    cells = nr * nt * np_
    ncomp = 3 if kind == "viscosity" else 1
    per_cell = {"A": b.alg_bytes_per_cell(ncomp)[0], "B": b.alg_bytes_per_cell(ncomp)[1],
                "Lpar": b.ANISO_BYTES_PER_CELL}[which]
    measured = d["dram_bytes_per_launch"] / cells
    assert 0.95 <= measured / per_cell <= 1.20, (prof, measured, per_cell)
    if "traffic_over_alg" in d:  # the stored ratio is per launch, not per cell
        assert abs(d["traffic_over_alg"] - measured / per_cell) < 1e-6


def test_config_shapes_follow_baseline():
    b = load_bench()
    cfgs = json.load(open(os.path.join(ROOT, "BASELINE.json")))["configs"]
    shapes = [tuple(int(v) for v in re.search(r"(\d+)\D(\d+)\D(\d+)", c).groups()) for c in cfgs]
    assert b.CONFIGS["C1"][1:] == shapes[0]
    assert b.CONFIGS["C2"][1:] == shapes[1]
    assert b.CONFIGS["C2a"][1:] == shapes[1]
    assert b.CONFIGS["C3"][1:] == shapes[2]
    assert b.CONFIGS["C4"][1:] == shapes[3]
    assert b.scaling_of("C4") == "weak" and b.scaling_of("C3") == "strong"
    # C3 is the ~36 M-cell headline grid of the metric
    assert 30e6 < shapes[2][0] * shapes[2][1] * shapes[2][2] < 40e6
