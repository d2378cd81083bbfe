"""Thin Python binding of the C ABI in include/mas_pcg.h (argument marshalling
only: every step of the solve runs in lib/libmaspcg.so's CUDA kernels).

Functions keep the C names (mas_grid_create, mas_op_setup, mas_op_apply,
mas_pcg_solve, ...) and accept torch tensors (CUDA or CPU) or numpy arrays;
they pass data pointers and the current torch CUDA stream.  There is no CPU
fallback: if the shared library is missing, import fails loudly.
"""
from __future__ import annotations

import ctypes as C
import os
from typing import Optional

import numpy as np

from . import build as _build

MAS_OK, MAS_NOT_CONVERGED, MAS_ERR_ARG, MAS_ERR_CUDA, MAS_ERR_NCCL, MAS_ERR_NOMEM, \
    MAS_ERR_BREAKDOWN = range(7)
MAS_BC_DIRICHLET, MAS_BC_NEUMANN = 0, 1
MAS_POLE_NORTH, MAS_POLE_SOUTH = 1, 2
MAS_PLACE_CELL, MAS_PLACE_THETA_NODE, MAS_PLACE_R_NODE, MAS_PLACE_PHI_NODE = 0, 1, 2, 3

# every symbol include/mas_pcg.h declares
ABI_SYMBOLS = ("mas_comm_unique_id", "mas_partition", "mas_grid_create", "mas_grid_local_extent",
               "mas_grid_destroy", "mas_op_setup", "mas_op_setup_placed", "mas_op_update", "mas_op_apply", "mas_op_diag",
               "mas_op_dirichlet_rhs", "mas_op_dot", "mas_pcg_solve", "mas_op_enable_p2p",
               "mas_op_transport", "mas_op_launch_count", "mas_grid_create_2d",
               "mas_grid_local_extent_2d",
               "mas_op_set_profiling", "mas_op_kernel_times", "mas_op_set_aniso",
               "mas_op_aniso_time", "mas_op_radial_sums", "mas_op_comm_bench", "mas_op_set_single_reduction", "mas_op_set_curvature", "mas_op_kernel_bench", "mas_op_aniso_fused",
               "mas_op_single_reduction", "mas_stack_create", "mas_stack_solve", "mas_stack_destroy",
               "mas_op_destroy", "mas_status_string", "mas_last_error", "mas_version")


class MasError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        super().__init__(f"{where}: {status_string(status)} ({detail})")
        self.status = status


class mas_dist_t(C.Structure):
    _fields_ = [("nranks", C.c_int), ("rank", C.c_int), ("nccl_id", C.c_ubyte * 128)]


_lib: Optional[C.CDLL] = None
_vp, _i, _d = C.c_void_p, C.c_int, C.c_double


def lib() -> C.CDLL:
    """Load lib/libmaspcg.so (never rebuilt here; see build.py / build())."""
    global _lib
    if _lib is None:
        if not os.path.exists(_build.SO):
            raise ImportError(f"{_build.SO} missing: run __graft_entry__.build() "
                              "(there is no CPU fallback)")
        L = C.CDLL(_build.SO)
        sig = {
            "mas_comm_unique_id": (_i, [_vp]),
            "mas_grid_create": (_i, [_i, _i, _i, _vp, _vp, _vp, _vp, _vp, _vp, _i, _i, _vp, _vp]),
            "mas_partition": (_i, [_i, _i, _i, _vp, _vp]),
            "mas_grid_local_extent": (_i, [_vp, _vp, _vp]),
            "mas_grid_create_2d": (_i, [_i, _i, _i, _vp, _vp, _vp, _vp, _vp, _vp, _i, _i, _vp, _i,
                                        _vp]),
            "mas_grid_local_extent_2d": (_i, [_vp, _vp, _vp, _vp, _vp]),
            "mas_grid_destroy": (_i, [_vp]),
            "mas_op_setup": (_i, [_vp, _i, _vp, _vp, _i, _i, _vp, _vp]),
            "mas_op_setup_placed": (_i, [_vp, _i, _i, _vp, _vp, _i, _i, _vp, _vp]),
            "mas_op_update": (_i, [_vp, _vp, _vp, _vp]),
            "mas_op_apply": (_i, [_vp, _vp, _vp, _vp]),
            "mas_op_diag": (_i, [_vp, _vp, _vp]),
            "mas_op_dirichlet_rhs": (_i, [_vp, _vp, _vp, _vp, _vp]),
            "mas_op_dot": (_i, [_vp, _vp, _vp, _vp, _vp]),
            "mas_pcg_solve": (_i, [_vp, _vp, _vp, _d, _i, _vp, _vp, _vp, _vp]),
            "mas_op_enable_p2p": (_i, [_vp, _vp]),
            "mas_op_transport": (_i, [_vp]),
            "mas_op_launch_count": (C.c_longlong, [_vp]),
            "mas_op_set_profiling": (_i, [_vp, _i]),
            "mas_op_kernel_times": (_i, [_vp, _vp, _vp, _vp]),
            "mas_op_set_aniso": (_i, [_vp, _vp, _vp, _vp]),
            "mas_op_aniso_time": (_i, [_vp, _vp]),
            "mas_op_radial_sums": (_i, [_vp, _vp, _vp, _vp, _vp]),
            "mas_op_comm_bench": (_i, [_vp, _i, _vp, _vp, _vp, _vp]),
            "mas_op_set_single_reduction": (_i, [_vp, _i]),
            "mas_op_set_curvature": (_i, [_vp, _i]),
            "mas_op_kernel_bench": (_i, [_vp, _i, _vp, _vp, _vp, _vp]),
            "mas_op_aniso_fused": (_i, [_vp]),
            "mas_op_single_reduction": (_i, [_vp]),
            "mas_stack_create": (_i, [_vp, _i, _vp]),
            "mas_stack_solve": (_i, [_vp, _vp, _vp, _d, _i, _vp, _vp, _vp, _vp]),
            "mas_stack_destroy": (_i, [_vp]),
            "mas_op_destroy": (_i, [_vp]),
            "mas_status_string": (C.c_char_p, [_i]),
            "mas_last_error": (C.c_char_p, []),
            "mas_version": (C.c_char_p, []),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype, f.argtypes = res, args
        _lib = L
    return _lib


def status_string(s: int) -> str:
    return lib().mas_status_string(s).decode()


def last_error() -> str:
    return lib().mas_last_error().decode()


def _check(s: int, where: str, ok=(MAS_OK,)) -> int:
    if s not in ok:
        raise MasError(s, where, last_error())
    return s


def _ptr(a) -> Optional[int]:
    """Data pointer of a torch tensor or numpy array (must be contiguous fp64,
    16-byte aligned: the kernels load double2 pairs and TMA boxes)."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        if a.dtype != np.float64 or not a.flags.c_contiguous:
            raise TypeError("need C-contiguous float64 arrays")
        p = a.ctypes.data
    else:
        import torch
        if not isinstance(a, torch.Tensor):
            raise TypeError(f"unsupported array type {type(a)}")
        if a.dtype != torch.float64 or not a.is_contiguous():
            raise TypeError("need contiguous float64 tensors")
        p = a.data_ptr()
    if p % 16:
        raise ValueError("array data must be 16-byte aligned (a view with an odd element "
                         "offset is not)")
    return p


def _numel(a) -> int:
    return int(a.size) if isinstance(a, np.ndarray) else int(a.numel())


def _expect(a, n: int, what: str) -> None:
    """The C side reads exactly n doubles (the LOCAL block on this rank)."""
    if a is not None and _numel(a) != n:
        raise ValueError(f"{what}: {_numel(a)} elements, the local block needs {n}")


def _stream(stream=None) -> Optional[int]:
    if stream is not None:
        return stream if isinstance(stream, int) else stream.cuda_stream
    import torch
    if torch.cuda.is_available():
        return torch.cuda.current_stream().cuda_stream
    return None


# ---------------------------------------------------------------------------
# C-named entry points
# ---------------------------------------------------------------------------
def mas_comm_unique_id() -> bytes:
    buf = (C.c_ubyte * 128)()
    _check(lib().mas_comm_unique_id(buf), "mas_comm_unique_id")
    return bytes(buf)


def virtual_ranks_id(key: int) -> bytes:
    """mas_dist_t.nccl_id selecting the in-process "virtual ranks" transport:
    P ranks as P host threads on one GPU (test transport, see comm.cpp; the
    library honours it only with MAS_TEST_TRANSPORTS=1 in the environment)."""
    return b"MASVIRT\0" + int(key).to_bytes(8, "little") + bytes(112)


def host_exchange_id(directory: str) -> bytes:
    """mas_dist_t.nccl_id selecting the "host exchange" test transport: P
    processes on ONE GPU exchange the setup-time collectives through files in
    `directory` (comm.cpp); the P2P loop then runs across real processes."""
    d = os.fsencode(directory)
    if len(d) > 119:
        raise ValueError("directory path too long (max 119 bytes)")
    return b"MASHOST\0" + d + bytes(120 - len(d))


def mas_grid_create(r_node, r_half, t_node, t_half, p_node, p_half, pole_flags=3,
                    periodic_phi=1, dist: Optional[tuple] = None, ptheta: int = 1) -> int:
    """dist = (nranks, rank, nccl_id_bytes) or None.  ptheta > 1: (r, theta)
    decomposition through mas_grid_create_2d.  Returns the handle."""
    arrs = [np.ascontiguousarray(a, dtype=np.float64) for a in
            (r_node, r_half, t_node, t_half, p_node, p_half)]
    nr, nt, np_ = len(arrs[1]), len(arrs[3]), len(arrs[5])
    for a, n in zip(arrs[::2], (nr, nt, np_)):
        if len(a) != n + 1:
            raise ValueError("node arrays must have n+1 entries")
    d = None
    if dist is not None:
        d = mas_dist_t(dist[0], dist[1])
        C.memmove(d.nccl_id, dist[2], 128)
    out = C.c_void_p()
    _check(lib().mas_grid_create_2d(nr, nt, np_, *[a.ctypes.data for a in arrs], pole_flags,
                                    periodic_phi, C.byref(d) if d is not None else None,
                                    int(ptheta), C.byref(out)), "mas_grid_create_2d")
    return out.value


def mas_grid_local_extent_2d(g: int):
    i0, nl, j0, ntl = C.c_int(), C.c_int(), C.c_int(), C.c_int()
    _check(lib().mas_grid_local_extent_2d(g, C.byref(i0), C.byref(nl), C.byref(j0), C.byref(ntl)),
           "mas_grid_local_extent_2d")
    return i0.value, nl.value, j0.value, ntl.value


def mas_partition(nr: int, nranks: int, rank: int):
    i0, nl = C.c_int(), C.c_int()
    _check(lib().mas_partition(nr, nranks, rank, C.byref(i0), C.byref(nl)), "mas_partition")
    return i0.value, nl.value


def mas_grid_local_extent(g: int):
    i0, nl = C.c_int(), C.c_int()
    _check(lib().mas_grid_local_extent(g, C.byref(i0), C.byref(nl)), "mas_grid_local_extent")
    return i0.value, nl.value


def mas_grid_destroy(g: int) -> None:
    _check(lib().mas_grid_destroy(g), "mas_grid_destroy")


def mas_op_setup(g: int, ncomp: int, kappa, mass=None, bc_r_inner=MAS_BC_DIRICHLET,
                 bc_r_outer=MAS_BC_NEUMANN, stream=None) -> int:
    out = C.c_void_p()
    _check(lib().mas_op_setup(g, ncomp, _ptr(kappa), _ptr(mass), bc_r_inner, bc_r_outer,
                              _stream(stream), C.byref(out)), "mas_op_setup")
    return out.value


def mas_op_setup_placed(g: int, ncomp: int, placement: int, kappa, mass=None,
                        bc_r_inner=MAS_BC_DIRICHLET, bc_r_outer=MAS_BC_NEUMANN, stream=None) -> int:
    """NEXT-2: placement MAS_PLACE_THETA_NODE puts the unknowns on the theta
    nodes (rows 0 and nt on the poles): arrays [comp][nl][nt+1][np]."""
    out = C.c_void_p()
    _check(lib().mas_op_setup_placed(g, ncomp, placement, _ptr(kappa), _ptr(mass), bc_r_inner,
                                     bc_r_outer, _stream(stream), C.byref(out)), "mas_op_setup_placed")
    return out.value


def mas_op_update(op: int, kappa, mass=None, stream=None) -> None:
    _check(lib().mas_op_update(op, _ptr(kappa), _ptr(mass), _stream(stream)), "mas_op_update")


def mas_op_apply(op: int, x, y, stream=None) -> None:
    _check(lib().mas_op_apply(op, _ptr(x), _ptr(y), _stream(stream)), "mas_op_apply")


def mas_op_diag(op: int, D, stream=None) -> None:
    _check(lib().mas_op_diag(op, _ptr(D), _stream(stream)), "mas_op_diag")


def mas_op_dirichlet_rhs(op: int, ub_inner, ub_outer, f, stream=None) -> None:
    _check(lib().mas_op_dirichlet_rhs(op, _ptr(ub_inner), _ptr(ub_outer), _ptr(f),
                                      _stream(stream)), "mas_op_dirichlet_rhs")


def mas_op_dot(op: int, a, b, stream=None) -> float:
    out = C.c_double()
    _check(lib().mas_op_dot(op, _ptr(a), _ptr(b), C.byref(out), _stream(stream)), "mas_op_dot")
    return out.value


def mas_pcg_solve(op: int, rhs, x, tol: float, maxit: int, want_hist: bool = False,
                  stream=None):
    """Returns (status, iters, relres, res_hist or None)."""
    it, rel = C.c_int(), C.c_double()
    hist = np.zeros(maxit + 1) if want_hist else None
    s = lib().mas_pcg_solve(op, _ptr(rhs), _ptr(x), float(tol), int(maxit), C.byref(it),
                            C.byref(rel), hist.ctypes.data if want_hist else None,
                            _stream(stream))
    _check(s, "mas_pcg_solve", ok=(MAS_OK, MAS_NOT_CONVERGED, MAS_ERR_BREAKDOWN))
    if hist is not None:
        n = it.value if s == MAS_ERR_BREAKDOWN else it.value + 1
        hist = hist[:n]
    return s, it.value, rel.value, hist


def mas_stack_create(ops) -> int:
    arr = (C.c_void_p * len(ops))(*ops)
    h = C.c_void_p()
    _check(lib().mas_stack_create(arr, len(ops), C.byref(h)), "mas_stack_create")
    return h.value


def mas_stack_solve(stack: int, rhs, x, tol: float, maxit: int, want_hist: bool = False, stream=None):
    """rhs, x: one device array per block.  Returns (status, iters, relres,
    res_hist or None) of the stacked vector."""
    if len(rhs) != len(x):
        raise ValueError("one rhs and one x per block")
    R = (C.c_void_p * len(rhs))(*[_ptr(a) for a in rhs])
    X = (C.c_void_p * len(x))(*[_ptr(a) for a in x])
    it, rel = C.c_int(), C.c_double()
    hist = np.zeros(maxit + 1) if want_hist else None
    s = lib().mas_stack_solve(stack, R, X, float(tol), int(maxit), C.byref(it), C.byref(rel),
                              hist.ctypes.data if want_hist else None, _stream(stream))
    _check(s, "mas_stack_solve", ok=(MAS_OK, MAS_NOT_CONVERGED, MAS_ERR_BREAKDOWN))
    if hist is not None:
        hist = hist[:it.value if s == MAS_ERR_BREAKDOWN else it.value + 1]
    return s, it.value, rel.value, hist


def mas_stack_destroy(stack: int) -> None:
    _check(lib().mas_stack_destroy(stack), "mas_stack_destroy")


def mas_op_enable_p2p(op: int, stream=None) -> None:
    """Collective: the op's PCG loop uses the P2P (NVLink peer-memory) transport."""
    _check(lib().mas_op_enable_p2p(op, _stream(stream)), "mas_op_enable_p2p")


def mas_op_transport(op: int) -> str:
    return {0: "nccl", 1: "p2p"}.get(int(lib().mas_op_transport(op)), "invalid")


def mas_op_launch_count(op: int) -> int:
    return int(lib().mas_op_launch_count(op))


def mas_op_set_profiling(op: int, on: bool) -> None:
    _check(lib().mas_op_set_profiling(op, int(bool(on))), "mas_op_set_profiling")


def mas_op_kernel_times(op: int):
    """(avg ms kernel A, avg ms kernel B, iterations averaged) of the last solve."""
    a, b, n = C.c_double(), C.c_double(), C.c_int()
    _check(lib().mas_op_kernel_times(op, C.byref(a), C.byref(b), C.byref(n)),
           "mas_op_kernel_times")
    return a.value, b.value, n.value


def mas_op_set_aniso(op: int, kpar, bhat, stream=None) -> None:
    """Field-aligned conduction term L_par (NEXT-4): kpar [nl,nt,np] and
    bhat [3,nl,nt,np] of the LOCAL r-slab at the lower cell corners (R25);
    kpar None switches it off."""
    _check(lib().mas_op_set_aniso(op, _ptr(kpar), _ptr(bhat), _stream(stream)),
           "mas_op_set_aniso")


def mas_op_aniso_time(op: int) -> float:
    ms = C.c_double()
    _check(lib().mas_op_aniso_time(op, C.byref(ms)), "mas_op_aniso_time")
    return ms.value


def mas_op_radial_sums(op: int, x, w, out, stream=None) -> None:
    """out[m][i] = sum_{j,k} w[j][k] x[m][i][j][k] (the paper's sum0)."""
    _check(lib().mas_op_radial_sums(op, _ptr(x), _ptr(w), _ptr(out), _stream(stream)),
           "mas_op_radial_sums")


def mas_op_comm_bench(op: int, reps: int = 20, stream=None):
    """(seam_us, allreduce_us, seam_bytes) per round of the NCCL loop's
    exchange steps on this op (collective)."""
    a, b, c = C.c_double(), C.c_double(), C.c_double()
    _check(lib().mas_op_comm_bench(op, int(reps), C.byref(a), C.byref(b), C.byref(c), _stream(stream)),
           "mas_op_comm_bench")
    return a.value, b.value, c.value


def mas_op_set_single_reduction(op: int, on: bool = True) -> None:
    """NEXT-1: the single-reduction (Chronopoulos-Gear) PCG loop on this op."""
    _check(lib().mas_op_set_single_reduction(op, int(bool(on))), "mas_op_set_single_reduction")


def mas_op_set_curvature(op: int, on: bool = True) -> None:
    """NEXT-2: the vector-Laplacian curvature terms of the 3-component operator."""
    _check(lib().mas_op_set_curvature(op, int(bool(on))), "mas_op_set_curvature")


def mas_op_kernel_bench(op: int, reps: int = 20, stream=None):
    """(kernel A or single-reduction kernel, kernel B, L_par) device ms per
    launch from back-to-back graph replays (clobbers the op's work vectors)."""
    a, b, c = C.c_double(), C.c_double(), C.c_double()
    _check(lib().mas_op_kernel_bench(op, int(reps), C.byref(a), C.byref(b), C.byref(c), _stream(stream)),
           "mas_op_kernel_bench")
    return a.value, b.value, c.value


def mas_op_single_reduction(op: int) -> bool:
    return int(lib().mas_op_single_reduction(op)) == 1


def mas_op_destroy(op: int) -> None:
    _check(lib().mas_op_destroy(op), "mas_op_destroy")


def mas_version() -> str:
    return lib().mas_version().decode()


# ---------------------------------------------------------------------------
# small RAII helpers over the same calls
# ---------------------------------------------------------------------------
class Grid:
    def __init__(self, mesh, dist=None, ptheta=1):
        # the pole flags are the mesh's own declaration; mas_grid_create rejects
        # a north flag with t_node[0] != 0 or a south flag with t_node[nt] != pi
        # (MAS_ERR_ARG), nothing is dropped silently here
        flags = (MAS_POLE_NORTH if getattr(mesh, "pole_north", True) else 0) | \
                (MAS_POLE_SOUTH if getattr(mesh, "pole_south", True) else 0)
        self.h = mas_grid_create(mesh.rF, mesh.rC, mesh.tF, mesh.tC, mesh.pF, mesh.pC, flags, 1,
                                 dist, ptheta)
        self.i0, self.nl, self.j0, self.ntl = mas_grid_local_extent_2d(self.h)
        self.shape = (len(mesh.rC), len(mesh.tC), len(mesh.pC))
        self.local_cells = self.nl * self.ntl * self.shape[2]

    def close(self):
        if self.h:
            mas_grid_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Operator:
    """Array arguments are the LOCAL block of this rank: [nl][ntl][np] for
    per-cell coefficients, [ncomp][nl][ntl][np] for vectors."""

    def __init__(self, grid: Grid, ncomp, kappa, mass, bc_inner, bc_outer, stream=None,
                 placement=MAS_PLACE_CELL):
        self.grid = grid
        self.ncomp = ncomp
        self.placement = placement
        # theta nodes (NEXT-2): nt + 1 rows, the first and last on the poles;
        # r nodes: nr - 1 planes (one rank)
        self.rows = grid.shape[1] + 1 if placement == MAS_PLACE_THETA_NODE else grid.ntl
        self.planes = grid.shape[0] - 1 if placement == MAS_PLACE_R_NODE else grid.nl
        self.N = self.planes * self.rows * grid.shape[2]
        _expect(kappa, self.N, "kappa")
        _expect(mass, self.N, "mass")
        self.h = mas_op_setup_placed(grid.h, ncomp, placement, kappa, mass, bc_inner, bc_outer, stream)

    def update(self, kappa, mass, stream=None):
        _expect(kappa, self.N, "kappa")
        _expect(mass, self.N, "mass")
        mas_op_update(self.h, kappa, mass, stream)

    def apply(self, x, y, stream=None):
        _expect(x, self.ncomp * self.N, "x")
        _expect(y, self.ncomp * self.N, "y")
        mas_op_apply(self.h, x, y, stream)

    def diag(self, D, stream=None):
        _expect(D, self.N, "D")
        mas_op_diag(self.h, D, stream)

    def dirichlet_rhs(self, ub_inner, ub_outer, f, stream=None):
        nb = self.ncomp * self.rows * self.grid.shape[2]
        _expect(ub_inner, nb, "ub_inner")
        _expect(ub_outer, nb, "ub_outer")
        _expect(f, self.ncomp * self.N, "f")
        mas_op_dirichlet_rhs(self.h, ub_inner, ub_outer, f, stream)

    def dot(self, a, b, stream=None):
        _expect(a, self.ncomp * self.N, "a")
        _expect(b, self.ncomp * self.N, "b")
        return mas_op_dot(self.h, a, b, stream)

    def solve(self, rhs, x, tol, maxit, want_hist=False, stream=None):
        _expect(rhs, self.ncomp * self.N, "rhs")
        _expect(x, self.ncomp * self.N, "x")
        return mas_pcg_solve(self.h, rhs, x, tol, maxit, want_hist, stream)

    def enable_p2p(self, stream=None):
        mas_op_enable_p2p(self.h, stream)

    @property
    def transport(self):
        return mas_op_transport(self.h)

    def set_profiling(self, on=True):
        mas_op_set_profiling(self.h, on)

    def kernel_times(self):
        return mas_op_kernel_times(self.h)

    def set_aniso(self, kpar, bhat, stream=None):
        """kpar [nl][nt][np] and bhat [3][nl][nt][np] (component-major): the
        local r-slab, at the lower cell corners (R25)."""
        _expect(kpar, self.N, "kpar")
        if kpar is not None:
            _expect(bhat, 3 * self.N, "bhat")
        mas_op_set_aniso(self.h, kpar, bhat, stream)

    def set_single_reduction(self, on=True):
        mas_op_set_single_reduction(self.h, on)

    def set_curvature(self, on=True):
        mas_op_set_curvature(self.h, on)

    @property
    def single_reduction(self):
        return mas_op_single_reduction(self.h)

    def kernel_bench(self, reps=20, stream=None):
        return mas_op_kernel_bench(self.h, reps, stream)

    def comm_bench(self, reps=20, stream=None):
        return mas_op_comm_bench(self.h, reps, stream)

    @property
    def aniso_fused(self):
        """True if the iteration's L_par runs inside kernel A (mas_op_aniso_fused)."""
        return int(lib().mas_op_aniso_fused(self.h)) == 1

    def aniso_time(self):
        return mas_op_aniso_time(self.h)

    def radial_sums(self, x, w, out, stream=None):
        _expect(x, self.ncomp * self.N, "x")
        _expect(w, self.rows * self.grid.shape[2], "w")
        _expect(out, self.ncomp * self.planes, "out")
        mas_op_radial_sums(self.h, x, w, out, stream)

    @property
    def launch_count(self):
        return mas_op_launch_count(self.h)

    def close(self):
        if self.h:
            mas_op_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Stack:
    """One PCG on the stacked vector of several operators (mas_stack_*; NEXT-2,
    reading R34): e.g. MAS's viscous step with v_r, v_theta, v_phi each at its
    staggered location.  Keeps the Operators alive; close() before them."""

    def __init__(self, ops):
        self.ops = list(ops)
        self.h = mas_stack_create([o.h for o in self.ops])

    def solve(self, rhs, x, tol, maxit, want_hist=False, stream=None):
        if len(rhs) != len(self.ops) or len(x) != len(self.ops):
            raise ValueError("one rhs and one x per operator of the stack")
        for o, r, xx in zip(self.ops, rhs, x):
            _expect(r, o.ncomp * o.N, "rhs")
            _expect(xx, o.ncomp * o.N, "x")
        return mas_stack_solve(self.h, rhs, x, tol, maxit, want_hist, stream)

    def close(self):
        if self.h:
            mas_stack_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
