#!/usr/bin/env python
"""Per-kernel SASS instruction-class summary of lib/libmaspcg.so (sm_100a):
cuobjdump -sass, opcodes counted per kernel and grouped into classes
(global / shared / TMA / bulk-prefetch / async-copy memory ops, fp64 math,
barriers and mbarrier ops).  Static counts (instructions in the binary), the
evidence that e.g. k_aniso uses TMA (UTMALDG) and mbarriers (SYNCS), kernel A
the bulk L2 prefetch (UBLKPF) and cp.async (LDGSTS), and no kernel uses tensor
cores (no HMMA/UTCMMA: the path is a memory-bound stencil).

  python tools/sass_summary.py [lib.so] > profiles/r2_sass_summary.json
"""
import collections
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CLASSES = {
    "global_load": ("LDG",), "global_store": ("STG",), "shared_load": ("LDS",),
    "shared_store": ("STS",), "async_copy_LDGSTS": ("LDGSTS",), "tma_UTMALDG": ("UTMALDG",),
    "tma_store_UTMASTG": ("UTMASTG",), "bulk_prefetch_UBLKPF": ("UBLKPF",),
    "mbarrier_SYNCS": ("SYNCS",), "barrier_BAR": ("BAR",), "fp64_DFMA": ("DFMA",),
    "fp64_DADD": ("DADD",), "fp64_DMUL": ("DMUL",), "shuffle_SHFL": ("SHFL",),
    "atomic": ("ATOM", "RED"), "tensor_core": ("HMMA", "UTCMMA", "UTCHMMA", "UTCQMMA", "IMMA"),
}


def demangle(name):
    try:
        return subprocess.run(["c++filt", name], capture_output=True, text=True).stdout.strip()
    except Exception:
        return name


def main():
    lib = sys.argv[1] if len(sys.argv) > 1 else os.path.join(
        ROOT, "paper_conf_ipps_caplansl23_b200", "lib", "libmaspcg.so")
    out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
    kernels = collections.OrderedDict()
    cur = None
    for ln in out.splitlines():
        m = re.match(r"\s*Function : (\S+)", ln)
        if m:
            cur = demangle(m.group(1))
            kernels[cur] = collections.Counter()
            continue
        m = re.match(r"\s*/\*[0-9a-f]+\*/\s+(@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)(\.[A-Z0-9_.]+)?", ln)
        if cur and m:
            kernels[cur][m.group(2)] += 1
    res = {}
    for k, cnt in kernels.items():
        cls = {c: sum(v for op, v in cnt.items() if any(op.startswith(p) for p in pre))
               for c, pre in CLASSES.items()}
        res[k] = {"instructions": sum(cnt.values()), "classes": {c: v for c, v in cls.items() if v}}
    json.dump({"lib": os.path.relpath(lib, ROOT), "arch": "sm_100a", "kernels": res}, sys.stdout, indent=1)
    print()


if __name__ == "__main__":
    main()
