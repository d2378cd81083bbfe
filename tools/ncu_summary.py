#!/usr/bin/env python
"""Summarise ncu output for profiles/ (run here, on the CPU box).

  python tools/ncu_summary.py launches <launches.csv>         # per-kernel share of the run
  python tools/ncu_summary.py report <file.ncu-rep> [alg_bytes_per_cell cells]
      # key metrics of one capture; traffic_over_alg = DRAM bytes of the launch
      # / (alg_bytes_per_cell * cells of that launch)
"""
import collections
import csv
import io
import json
import subprocess
import sys


def launches(path):
    rows = list(csv.reader(open(path)))
    # find header line
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    h = rows[start]
    ik, im, iv = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
    agg = collections.OrderedDict()
    for r in rows[start + 1:]:
        if len(r) <= iv or r[im] != "gpu__time_duration.sum":
            continue
        name = r[ik].split("(")[0]
        t = float(r[iv].replace(",", ""))
        unit = r[h.index("Metric Unit")] if "Metric Unit" in h else "nsecond"
        scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(unit, 1e-3)
        c, s = agg.get(name, (0, 0.0))
        agg[name] = (c + 1, s + t * scale)
    tot = sum(s for _, s in agg.values())
    out = []
    for name, (c, s) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        out.append({"kernel": name, "launches": c, "total_us": round(s, 1), "avg_us": round(s / c, 2),
                    "share": round(s / tot, 4)})
    return {"total_us": round(tot, 1), "kernels": out}


KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_active",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
    "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem", "launch__grid_size",
    "launch__block_size", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "sm__cycles_elapsed.avg.per_second",
]
UNITS = {"dram__bytes_read.sum": "byte", "dram__bytes_write.sum": "byte"}


def report(path, alg_bytes=None):
    """alg_bytes: ALGORITHMIC bytes of the whole captured launch (per-cell
    figure x cells), never a per-cell figure."""
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, units, v = rows[0], rows[1], rows[2]
    d = dict(zip(h, v))
    u = dict(zip(h, units))
    out = {"kernel": d.get("Kernel Name"), "metrics": {}}
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    for k in KEYS:
        if k in d:
            val = d[k].replace(",", "")
            try:
                val = float(val)
            except ValueError:
                pass
            if k in UNITS and isinstance(val, float):
                val = val * scale.get(u[k], 1)
            out["metrics"][k] = val
            out.setdefault("units", {})[k] = u[k]
    stalls = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(d[k])
              for k in h if k.startswith("smsp__pcsamp_warps_issue_stalled_")
              and not k.endswith("_not_issued") and d[k] not in ("", "n/a")}
    tot = sum(stalls.values()) or 1.0
    out["stall_share"] = {k: round(s / tot, 3) for k, s in sorted(stalls.items(), key=lambda kv: -kv[1])
                          if s / tot > 0.02}
    m = out["metrics"]
    rd, wr = m.get("dram__bytes_read.sum"), m.get("dram__bytes_write.sum")
    if isinstance(rd, float) and isinstance(wr, float):
        out["dram_bytes_per_launch"] = rd + wr
        if alg_bytes:
            ratio = (rd + wr) / alg_bytes
            if not 0.05 < ratio < 20.0:
                raise SystemExit(f"traffic/alg = {ratio:.3g}: alg_bytes must be per launch "
                                 "(bytes per cell x cells), not per cell")
            out["alg_bytes_per_launch"] = alg_bytes
            out["traffic_over_alg"] = ratio
    return out


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        print(json.dumps(launches(sys.argv[2]), indent=1))
    else:
        alg = float(sys.argv[3]) * float(sys.argv[4]) if len(sys.argv) > 4 else None
        print(json.dumps(report(sys.argv[2], alg), indent=1))
