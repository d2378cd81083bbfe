"""CPU checks of bench.py's reported-figure helpers:
the algorithmic bytes per cell that the roofline objects divide by, and the
configs' shapes (BASELINE.json configs[1..3] sizes)."""
import importlib.util
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def load_bench():
    spec = importlib.util.spec_from_file_location("bench", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def test_algorithmic_bytes():
    b = load_bench()
    # kernel A: r, p_old, x (ncomp each) + D^-1, kappa, c read; p, q, x written
    # kernel B: r, q (ncomp) + D^-1 read; r written
    assert b.alg_bytes_per_cell(3) == (168, 80)  # 248 B per cell-iteration (C3)
    assert b.alg_bytes_per_cell(1) == (72, 32)   # 104 B (C2)
    assert b.ANISO_BYTES_PER_CELL == 48          # p + (a, b, e) read, q read + written
    assert b.oracle_bytes_per_cell(1) == 8 * 21


def test_config_shapes_follow_baseline():
    b = load_bench()
    assert b.CONFIGS["C3"][1:] == (256, 256, 512)
    assert b.CONFIGS["C2"][1:] == (128, 128, 256)
    assert b.CONFIGS["C2a"][1:] == (128, 128, 256)
    assert b.CONFIGS["C1"][1:] == (16, 24, 32)
    assert b.scaling_of("C4") == "weak" and b.scaling_of("C3") == "strong"
