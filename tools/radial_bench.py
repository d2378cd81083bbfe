"""Time mas_op_radial_sums (the paper's sum0) at the C3 size: GB/s of the
x read (ncomp * cells * 8 B per call) against the measured HBM copy peak."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_caplansl23_b200 import maspcg as M  # noqa: E402
from paper_conf_ipps_caplansl23_b200 import workloads as W  # noqa: E402

nr, nt, np_, nc = 256, 256, 512, 3
mesh = W.stretched_mesh(nr, nt, np_)
g = M.Grid(mesh)
op = M.Operator(g, nc, torch.ones((nr, nt, np_), dtype=torch.float64, device="cuda"), None, 0, 1)
x = torch.randn((nc, nr, nt, np_), dtype=torch.float64, device="cuda")
w = torch.randn((nt, np_), dtype=torch.float64, device="cuda")
out = torch.empty((nc, nr), dtype=torch.float64, device="cuda")
for _ in range(3):
    op.radial_sums(x, w, out)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
n = 20
e0.record()
for _ in range(n):
    op.radial_sums(x, w, out)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / n
gbs = nc * nr * nt * np_ * 8 / (ms / 1e3) / 1e9
peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                   "MEASURED_PEAKS.json"))).get("hbm_gbs", 6552.0)
print(json.dumps({"kernel": "k_radial_sums", "ms": ms, "GBs": gbs, "frac": gbs / peak}))
