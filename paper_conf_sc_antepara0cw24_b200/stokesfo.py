"""Thin ctypes binding of libstokesfo.so (include/stokesfo.h).

Argument marshalling only: every step of the evaluation runs in the library's
CUDA kernels.  PyTorch supplies device memory (tensors -> data_ptr()) and the
stream; nothing here computes the method.  There is no CPU fallback: if the
library cannot be loaded, every call raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import build as _build

HEX8, WEDGE6 = 0, 1
ELEM = {"hex8": HEX8, "wedge6": WEDGE6}
NODES = {HEX8: 8, WEDGE6: 6}
QPS = {HEX8: 8, WEDGE6: 6}
ABI_VERSION = 1

GEOMETRY = {"stored": 0, "on_the_fly": 1, "compact": 2}
STATUS = {0: "OK", 1: "EINVAL", 2: "EMESH", 3: "ECUDA", 4: "ENOMEM", 5: "EUNSUPPORTED", 6: "ENONFINITE"}


class StokesFOError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = _lib().stokesfo_strerror(status).decode() if _LIB is not None else STATUS.get(status, "?")
        super().__init__(f"{where}: {STATUS.get(status, status)} ({msg})")


class Desc(ctypes.Structure):
    _fields_ = [
        ("abi_version", ctypes.c_uint32), ("elem", ctypes.c_int32),
        ("num_cells", ctypes.c_int64), ("num_nodes", ctypes.c_int64),
        ("conn", ctypes.c_void_p), ("coords", ctypes.c_void_p), ("surface", ctypes.c_void_p),
        ("force_qp", ctypes.c_void_p), ("flow_factor", ctypes.c_void_p),
        ("k", ctypes.c_double), ("glen_n", ctypes.c_double), ("delta", ctypes.c_double),
        ("rho_g", ctypes.c_double),
        ("workspace", ctypes.c_void_p), ("workspace_bytes", ctypes.c_size_t),
        ("stream", ctypes.c_void_p),
        ("geometry_mode", ctypes.c_int32), ("reserved0", ctypes.c_int32),
    ]


_LIB = None
EXPORTS = [
    "stokesfo_workspace_size", "stokesfo_create", "stokesfo_gather", "stokesfo_viscosity_resid",
    "stokesfo_jacobian", "stokesfo_scatter_assemble", "stokesfo_csr_pattern", "stokesfo_geometry",
    "stokesfo_halo_pack", "stokesfo_halo_unpack_add", "stokesfo_sync", "stokesfo_strerror",
    "stokesfo_destroy", "stokesfo_launch_info", "stokesfo_mesh_extrude",
    "stokesfo_mesh_partition_columns", "stokesfo_mesh_localize", "stokesfo_mesh_halo_list",
    "stokesfo_albany_scratch_size", "stokesfo_albany_setup", "stokesfo_albany_evaluators",
    "stokesfo_albany_resid", "stokesfo_albany_extract", "stokesfo_jvp", "stokesfo_basal_friction",
    "stokesfo_set_remote", "stokesfo_set_remote_jvp", "stokesfo_ipc_get_handle", "stokesfo_ipc_open_handle", "stokesfo_ipc_close",
    "stokesfo_newton_work_size", "stokesfo_newton_solve", "stokesfo_lateral_pressure",
    "stokesfo_mesh_lateral_faces", "stokesfo_set_lateral", "stokesfo_csr_slots_size", "stokesfo_csr_slots", "stokesfo_jacobian_csr",
    "stokesfo_jacobian_diag", "stokesfo_assemble_csr", "stokesfo_jacobian_packed", "stokesfo_assemble_csr_packed",
]


class NewtonOpts(ctypes.Structure):
    _fields_ = [("max_newton", ctypes.c_int32), ("max_cg", ctypes.c_int32), ("max_ls", ctypes.c_int32),
                ("reserved", ctypes.c_int32), ("rtol_newton", ctypes.c_double), ("atol_newton", ctypes.c_double),
                ("rtol_cg", ctypes.c_double), ("ls_c", ctypes.c_double)]
FIG2 = {"baseline": 0, "optimized": 1}


def lib_path() -> str:
    # STOKESFO_LIB: load another build of the same ABI (same-box A/B measurements)
    return os.environ.get("STOKESFO_LIB", _build.LIB)


def _lib():
    """Load libstokesfo.so (building it in-tree with nvcc if absent)."""
    global _LIB
    if _LIB is None:
        path = lib_path()
        if path == _build.LIB and not os.path.exists(path):
            _build.build()
        L = ctypes.CDLL(path)
        P, I64, I32, D = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_double
        L.stokesfo_workspace_size.argtypes = [ctypes.POINTER(Desc), ctypes.POINTER(ctypes.c_size_t)]
        L.stokesfo_create.argtypes = [ctypes.POINTER(Desc), ctypes.POINTER(ctypes.c_void_p)]
        L.stokesfo_gather.argtypes = [P, P, P]
        L.stokesfo_viscosity_resid.argtypes = [P, P, P, P, P]
        L.stokesfo_jacobian.argtypes = [P, P, P, P, P]
        if hasattr(L, "stokesfo_jvp"):  # absent only in older builds loaded via STOKESFO_LIB
            L.stokesfo_jvp.argtypes = [P, P, P, P, P]
        if hasattr(L, "stokesfo_jacobian_diag"):
            L.stokesfo_jacobian_diag.argtypes = [P, P, P, P]
        if hasattr(L, "stokesfo_assemble_csr"):
            L.stokesfo_assemble_csr.argtypes = [P, P, P, ctypes.c_int]
        if hasattr(L, "stokesfo_jacobian_packed"):
            L.stokesfo_jacobian_packed.argtypes = [P, P, P, P, P]
            L.stokesfo_assemble_csr_packed.argtypes = [P, P, P, ctypes.c_int]
        if hasattr(L, "stokesfo_basal_friction"):
            L.stokesfo_basal_friction.argtypes = [P, P, I64, P, P, P, P]
        if hasattr(L, "stokesfo_lateral_pressure"):
            L.stokesfo_lateral_pressure.argtypes = [P, P, I64, P, D, D, D, P]
            L.stokesfo_mesh_lateral_faces.argtypes = [I32, I64, P, I32, ctypes.POINTER(I64), P]
            L.stokesfo_set_lateral.argtypes = [P, P, I64, P, D, D, D]
        if hasattr(L, "stokesfo_jacobian_csr"):
            L.stokesfo_csr_slots_size.argtypes = [P, ctypes.POINTER(ctypes.c_size_t)]
            L.stokesfo_csr_slots.argtypes = [P, P]
            L.stokesfo_jacobian_csr.argtypes = [P, P, P, P]
        if hasattr(L, "stokesfo_newton_solve"):
            L.stokesfo_newton_work_size.argtypes = [P, I64, ctypes.POINTER(ctypes.c_size_t)]
            L.stokesfo_newton_solve.argtypes = [P, P, I64, P, P, P, ctypes.POINTER(NewtonOpts), P, P,
                                                ctypes.POINTER(I32)]
        if hasattr(L, "stokesfo_set_remote"):
            L.stokesfo_set_remote.argtypes = [P, P, P, P]
            if hasattr(L, "stokesfo_set_remote_jvp"):
                L.stokesfo_set_remote_jvp.argtypes = [P, P]
            L.stokesfo_ipc_get_handle.argtypes = [P, P, ctypes.POINTER(I64)]
            L.stokesfo_ipc_open_handle.argtypes = [P, ctypes.POINTER(ctypes.c_void_p)]
            L.stokesfo_ipc_close.argtypes = [P]
        L.stokesfo_scatter_assemble.argtypes = [P, P, P, P, P]
        L.stokesfo_csr_pattern.argtypes = [P, ctypes.POINTER(I64), P, P]
        L.stokesfo_geometry.argtypes = [P, P, P]
        L.stokesfo_halo_pack.argtypes = [P, P, P, I64, P]
        L.stokesfo_halo_unpack_add.argtypes = [P, P, P, I64, P]
        L.stokesfo_sync.argtypes = [P]
        L.stokesfo_strerror.argtypes = [ctypes.c_int]
        L.stokesfo_strerror.restype = ctypes.c_char_p
        L.stokesfo_destroy.argtypes = [P]
        L.stokesfo_destroy.restype = None
        L.stokesfo_launch_info.argtypes = [P, ctypes.POINTER(I32), ctypes.POINTER(I32), ctypes.POINTER(I32),
                                           ctypes.POINTER(I64)]
        L.stokesfo_mesh_extrude.argtypes = [I32, I64, P, I64, P, P, P, I32, P, P]
        L.stokesfo_mesh_partition_columns.argtypes = [I64, I32, P]
        L.stokesfo_mesh_localize.argtypes = [I32, I64, P, ctypes.POINTER(I64), P, P]
        L.stokesfo_mesh_halo_list.argtypes = [I64, P, I64, P, ctypes.POINTER(I64), P]
        L.stokesfo_albany_scratch_size.argtypes = [P, ctypes.c_int, ctypes.POINTER(ctypes.c_size_t)]
        L.stokesfo_albany_setup.argtypes = [P, ctypes.c_int, P]
        L.stokesfo_albany_evaluators.argtypes = [P, ctypes.c_int, P, P]
        L.stokesfo_albany_resid.argtypes = [P, ctypes.c_int, ctypes.c_int, P]
        L.stokesfo_albany_extract.argtypes = [P, ctypes.c_int, P, P, P]
        _LIB = L
    return _LIB


def _check(st: int, where: str):
    if st != 0:
        raise StokesFOError(st, where)


def _ptr(t):
    """Device (or host numpy) pointer of a tensor/array, or None."""
    if t is None:
        return None
    if isinstance(t, np.ndarray):
        return t.ctypes.data_as(ctypes.c_void_p)
    return ctypes.c_void_p(t.data_ptr())


def _dev(t, dtype, shape=None, name="array"):
    import torch
    if t is None:
        return None
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA tensor")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    if shape is not None and tuple(t.shape) != tuple(shape):
        raise ValueError(f"{name} must have shape {tuple(shape)}, got {tuple(t.shape)}")
    return t


class StokesFO:
    """One evaluation context (stokesfo_ctx) over a local mesh on one GPU."""

    def __init__(self, elem, conn, coords, surface=None, force_qp=None, flow_factor=None, k=10.77,
                 glen_n=3.0, delta=1e-10, rho_g=8.927, stream=None, geometry="stored"):
        import torch
        self.elem = ELEM[elem] if isinstance(elem, str) else int(elem)
        self.N, self.Q = NODES[self.elem], QPS[self.elem]
        C = int(conn.shape[0])
        nn = int(coords.shape[0])
        self.num_cells, self.num_nodes = C, nn
        self.conn = _dev(conn, torch.int32, (C, self.N), "conn")
        self.coords = _dev(coords, torch.float64, (nn, 3), "coords")
        self.surface = _dev(surface, torch.float64, (nn,), "surface")
        self.force_qp = _dev(force_qp, torch.float64, (C, self.Q, 2), "force_qp")
        self.flow_factor = _dev(flow_factor, torch.float64, (C,), "flow_factor")
        self.device = self.coords.device
        self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
        d = Desc()
        d.abi_version = ABI_VERSION
        d.elem = self.elem
        d.num_cells, d.num_nodes = C, nn
        d.conn, d.coords = _ptr(self.conn), _ptr(self.coords)
        d.surface, d.force_qp, d.flow_factor = _ptr(self.surface), _ptr(self.force_qp), _ptr(self.flow_factor)
        d.k, d.glen_n, d.delta, d.rho_g = k, glen_n, delta, rho_g
        d.stream = ctypes.c_void_p(self.stream.cuda_stream)
        self.geometry_mode = GEOMETRY[geometry] if isinstance(geometry, str) else int(geometry)
        d.geometry_mode = self.geometry_mode
        nbytes = ctypes.c_size_t(0)
        _check(_lib().stokesfo_workspace_size(ctypes.byref(d), ctypes.byref(nbytes)), "workspace_size")
        self.workspace = torch.empty(max(int(nbytes.value), 256), dtype=torch.uint8, device=self.device)
        d.workspace, d.workspace_bytes = _ptr(self.workspace), self.workspace.numel()
        self._desc = d
        h = ctypes.c_void_p()
        _check(_lib().stokesfo_create(ctypes.byref(d), ctypes.byref(h)), "create")
        self._h = h
        self.rowptr = None
        self.colidx = None

    # -- lifetime -------------------------------------------------------------
    def destroy(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            _lib().stokesfo_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass

    # -- calls (same names as the C ABI) --------------------------------------
    def gather(self, U, U_cell=None):
        import torch
        _dev(U, torch.float64, (self.num_nodes, 2), "U")
        if U_cell is None:
            U_cell = torch.empty((self.num_cells, self.N, 2), dtype=torch.float64, device=self.device)
        _check(_lib().stokesfo_gather(self._h, _ptr(U), _ptr(U_cell)), "gather")
        return U_cell

    def viscosity_resid(self, U, mu_qp=None, R_cell=None, R=None):
        import torch
        _dev(U, torch.float64, (self.num_nodes, 2), "U")
        _dev(mu_qp, torch.float64, (self.num_cells, self.Q), "mu_qp")
        _dev(R_cell, torch.float64, (self.num_cells, self.N, 2), "R_cell")
        _dev(R, torch.float64, (self.num_nodes, 2), "R")
        _check(_lib().stokesfo_viscosity_resid(self._h, _ptr(U), _ptr(mu_qp), _ptr(R_cell), _ptr(R)),
               "viscosity_resid")

    def jacobian(self, U, J_cell, R_cell=None, R=None):
        import torch
        _dev(U, torch.float64, (self.num_nodes, 2), "U")
        _dev(J_cell, torch.float64, (self.num_cells, 2 * self.N, 2 * self.N), "J_cell")
        _dev(R_cell, torch.float64, (self.num_cells, self.N, 2), "R_cell")
        _dev(R, torch.float64, (self.num_nodes, 2), "R")
        _check(_lib().stokesfo_jacobian(self._h, _ptr(U), _ptr(J_cell), _ptr(R_cell), _ptr(R)), "jacobian")

    def jvp(self, U, X, Y, R=None):
        """Y += J(U) X (matrix-free, no element matrices); optionally R += R(U)."""
        import torch
        for t, n in ((U, "U"), (X, "X"), (Y, "Y")):
            _dev(t, torch.float64, (self.num_nodes, 2), n)
        _dev(R, torch.float64, (self.num_nodes, 2), "R")
        _check(_lib().stokesfo_jvp(self._h, _ptr(U), _ptr(X), _ptr(Y), _ptr(R)), "jvp")

    def jacobian_diag(self, U, diag, R=None):
        """diag += diagonal of the assembled Jacobian J(U) (no element matrices); optionally R += R(U)."""
        import torch
        for t, n in ((U, "U"), (diag, "diag")):
            _dev(t, torch.float64, (self.num_nodes, 2), n)
        _dev(R, torch.float64, (self.num_nodes, 2), "R")
        _check(_lib().stokesfo_jacobian_diag(self._h, _ptr(U), _ptr(diag), _ptr(R)), "jacobian_diag")

    def basal_friction(self, basal_cells, beta, U, R, J_face=None):
        """R += basal friction term on the bottom faces of basal_cells (int32 cuda);
        optional J_face [nfaces][2NB][2NB] (NB = 4 hex8 / 3 wedge6)."""
        import torch
        _dev(basal_cells, torch.int32, None, "basal_cells")
        _dev(beta, torch.float64, (self.num_nodes,), "beta")
        _dev(U, torch.float64, (self.num_nodes, 2), "U")
        _dev(R, torch.float64, (self.num_nodes, 2), "R")
        _check(_lib().stokesfo_basal_friction(self._h, _ptr(basal_cells), int(basal_cells.numel()), _ptr(beta),
                                              _ptr(U), _ptr(R), _ptr(J_face)), "basal_friction")

    def lateral_pressure(self, faces, surface, R, rho_i_g=8.927, rho_w_g=10.05, sea_level=0.0):
        """R -= lateral (calving-front) pressure term on faces (int32 cuda [nfaces][2] = (cell, side))."""
        import torch
        _dev(faces, torch.int32, None, "faces")
        if faces.dim() != 2 or faces.shape[1] != 2:
            raise ValueError("faces must have shape [nfaces][2]")
        _dev(surface, torch.float64, (self.num_nodes,), "surface")
        _dev(R, torch.float64, (self.num_nodes, 2), "R")
        _check(_lib().stokesfo_lateral_pressure(self._h, _ptr(faces), int(faces.shape[0]), _ptr(surface),
                                                float(rho_i_g), float(rho_w_g), float(sea_level), _ptr(R)),
               "lateral_pressure")

    def set_lateral(self, faces, surface, rho_i_g=8.927, rho_w_g=10.05, sea_level=0.0):
        """Attach the lateral pressure term to newton_solve's F (faces=None detaches)."""
        import torch
        if faces is None:
            self._lateral_keep = None
            _check(_lib().stokesfo_set_lateral(self._h, None, 0, None, 0.0, 0.0, 0.0), "set_lateral")
            return
        _dev(faces, torch.int32, None, "faces")
        _dev(surface, torch.float64, (self.num_nodes,), "surface")
        self._lateral_keep = (faces, surface)
        _check(_lib().stokesfo_set_lateral(self._h, _ptr(faces), int(faces.shape[0]), _ptr(surface), float(rho_i_g),
                                           float(rho_w_g), float(sea_level)), "set_lateral")

    def newton_solve(self, basal_cells, beta, U, max_newton=8, max_cg=500, max_ls=20, rtol_newton=1e-10,
                     atol_newton=0.0, rtol_cg=1e-6, ls_c=1e-4):
        """Damped Newton-Krylov solve of R_visc(U) + R_basal(U) = 0 in place on U
        (stokesfo_newton_solve).  Returns {"F": [||F_k||], "cg": [iters], "iters": k}."""
        import torch
        _dev(U, torch.float64, (self.num_nodes, 2), "U")
        nb = 0 if basal_cells is None else int(basal_cells.numel())
        n = ctypes.c_size_t(0)
        _check(_lib().stokesfo_newton_work_size(self._h, nb, ctypes.byref(n)), "newton_work_size")
        work = torch.empty(int(n.value), dtype=torch.uint8, device=self.device)
        o = NewtonOpts(max_newton, max_cg, max_ls, 0, rtol_newton, atol_newton, rtol_cg, ls_c)
        hF = (ctypes.c_double * (max_newton + 1))()
        hc = (ctypes.c_int32 * max(max_newton, 1))()
        it = ctypes.c_int32(0)
        _check(_lib().stokesfo_newton_solve(self._h, _ptr(basal_cells), nb, _ptr(beta), _ptr(U), _ptr(work),
                                            ctypes.byref(o), hF, hc, ctypes.byref(it)), "newton_solve")
        k = it.value
        return {"F": [hF[i] for i in range(k + 1)], "cg": [hc[i] for i in range(k)], "iters": k}

    def set_remote(self, rem, remtab, peers):
        """Fused halo over peer memory (stokesfo_set_remote); rem=None detaches."""
        self._remote_keep = (rem, remtab, peers)
        _check(_lib().stokesfo_set_remote(self._h, _ptr(rem), _ptr(remtab), _ptr(peers)), "set_remote")
        if rem is None:
            self._remote_y_keep = None

    def set_remote_jvp(self, peers_y):
        """The peers' J.v outputs for jvp under the attached node table (stokesfo_set_remote_jvp)."""
        self._remote_y_keep = peers_y
        _check(_lib().stokesfo_set_remote_jvp(self._h, _ptr(peers_y)), "set_remote_jvp")

    def csr_pattern(self):
        import torch
        nnz = ctypes.c_int64(0)
        _check(_lib().stokesfo_csr_pattern(self._h, ctypes.byref(nnz), None, None), "csr_pattern(size)")
        self.rowptr = torch.empty(2 * self.num_nodes + 1, dtype=torch.int64, device=self.device)
        self.colidx = torch.empty(max(int(nnz.value), 1), dtype=torch.int32, device=self.device)
        _check(_lib().stokesfo_csr_pattern(self._h, ctypes.byref(nnz), _ptr(self.rowptr), _ptr(self.colidx)),
               "csr_pattern")
        self.colidx = self.colidx[:int(nnz.value)]
        return self.rowptr, self.colidx

    def csr_slots(self):
        """Per-cell CSR slot table (stokesfo_csr_slots); needs csr_pattern() first."""
        import torch
        n = ctypes.c_size_t(0)
        _check(_lib().stokesfo_csr_slots_size(self._h, ctypes.byref(n)), "csr_slots_size")
        self.slots = torch.empty(max(int(n.value) // 8, 2), dtype=torch.int64, device=self.device)
        _check(_lib().stokesfo_csr_slots(self._h, _ptr(self.slots)), "csr_slots")
        C, N = self.num_cells, self.N
        return self.slots[:C * N]

    def jacobian_csr(self, U, csr_vals, R=None):
        """csr_vals += assembled Jacobian (fused, no element matrices); optionally R += residual."""
        import torch
        _dev(U, torch.float64, (self.num_nodes, 2), "U")
        _dev(csr_vals, torch.float64, None, "csr_vals")
        _dev(R, torch.float64, (self.num_nodes, 2), "R")
        _check(_lib().stokesfo_jacobian_csr(self._h, _ptr(U), _ptr(csr_vals), _ptr(R)), "jacobian_csr")

    def assemble_csr(self, J_cell, csr_vals, accumulate=False):
        """csr_vals (+)= the global matrix assembled from element matrices (stokesfo_assemble_csr;
        pull assembly, after csr_slots); accumulate=False overwrites every entry."""
        _check(_lib().stokesfo_assemble_csr(self._h, _ptr(J_cell), _ptr(csr_vals), 1 if accumulate else 0),
               "assemble_csr")

    @property
    def packed_blocks(self):
        """N(N+1)/2: upper 2 x 2 node blocks per cell of the symmetric block-packed element matrix."""
        return self.N * (self.N + 1) // 2

    def jacobian_packed(self, U, Jp, R_cell=None, R=None):
        """Element Jacobians in symmetric block-packed form Jp [C][N(N+1)/2][2][2] (stokesfo_jacobian_packed)."""
        import torch
        _dev(U, torch.float64, (self.num_nodes, 2), "U")
        _dev(Jp, torch.float64, (self.num_cells, self.packed_blocks, 2, 2), "Jp")
        _dev(R_cell, torch.float64, (self.num_cells, self.N, 2), "R_cell")
        _dev(R, torch.float64, (self.num_nodes, 2), "R")
        _check(_lib().stokesfo_jacobian_packed(self._h, _ptr(U), _ptr(Jp), _ptr(R_cell), _ptr(R)), "jacobian_packed")

    def assemble_csr_packed(self, Jp, csr_vals, accumulate=False):
        """csr_vals (+)= the global matrix assembled from packed element matrices (stokesfo_assemble_csr_packed)."""
        _check(_lib().stokesfo_assemble_csr_packed(self._h, _ptr(Jp), _ptr(csr_vals), 1 if accumulate else 0),
               "assemble_csr_packed")

    def scatter_assemble(self, R_cell=None, R=None, J_cell=None, csr_vals=None):
        _check(_lib().stokesfo_scatter_assemble(self._h, _ptr(R_cell), _ptr(R), _ptr(J_cell), _ptr(csr_vals)),
               "scatter_assemble")

    def geometry(self):
        import torch
        G = torch.empty((self.num_cells, self.N, self.Q, 3), dtype=torch.float64, device=self.device)
        wm = torch.empty((self.num_cells, self.Q), dtype=torch.float64, device=self.device)
        _check(_lib().stokesfo_geometry(self._h, _ptr(G), _ptr(wm)), "geometry")
        return G, wm

    def halo_pack(self, R, send_nodes, buf):
        _check(_lib().stokesfo_halo_pack(self._h, _ptr(R), _ptr(send_nodes), int(send_nodes.numel()), _ptr(buf)),
               "halo_pack")

    def halo_unpack_add(self, buf, recv_nodes, R):
        _check(_lib().stokesfo_halo_unpack_add(self._h, _ptr(buf), _ptr(recv_nodes), int(recv_nodes.numel()),
                                               _ptr(R)), "halo_unpack_add")

    def sync(self):
        _check(_lib().stokesfo_sync(self._h), "sync")

    # -- NEXT-1: the paper's evaluator chain (baseline / optimized Fig. 2) -----
    def albany_scratch(self, derivs: bool):
        import torch
        n = ctypes.c_size_t(0)
        _check(_lib().stokesfo_albany_scratch_size(self._h, int(derivs), ctypes.byref(n)), "albany_scratch_size")
        return torch.empty(max(int(n.value) // 8, 1), dtype=torch.float64, device=self.device)

    def albany_setup(self, derivs: bool, scratch):
        _check(_lib().stokesfo_albany_setup(self._h, int(derivs), _ptr(scratch)), "albany_setup")

    def albany_evaluators(self, derivs: bool, U, scratch):
        _check(_lib().stokesfo_albany_evaluators(self._h, int(derivs), _ptr(U), _ptr(scratch)), "albany_evaluators")

    def albany_resid(self, derivs: bool, variant, scratch):
        v = FIG2[variant] if isinstance(variant, str) else int(variant)
        _check(_lib().stokesfo_albany_resid(self._h, int(derivs), v, _ptr(scratch)), "albany_resid")

    def albany_extract(self, derivs: bool, scratch, R_cell=None, J_cell=None):
        _check(_lib().stokesfo_albany_extract(self._h, int(derivs), _ptr(scratch), _ptr(R_cell), _ptr(J_cell)),
               "albany_extract")

    def launch_info(self):
        tc, gr, gj = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int32()
        rb = ctypes.c_int64()
        _check(_lib().stokesfo_launch_info(self._h, ctypes.byref(tc), ctypes.byref(gr), ctypes.byref(gj),
                                           ctypes.byref(rb)), "launch_info")
        return {"cells_per_tile": tc.value, "grid_resid": gr.value, "grid_jac": gj.value,
                "record_bytes_per_tile": rb.value}


def ipc_get_handle(t):
    """(64-byte CUDA IPC handle of the tensor's allocation, offset of the tensor in it)."""
    buf = ctypes.create_string_buffer(64)
    off = ctypes.c_int64(0)
    _check(_lib().stokesfo_ipc_get_handle(ctypes.c_void_p(t.data_ptr()), buf, ctypes.byref(off)), "ipc_get_handle")
    return buf.raw, int(off.value)


def ipc_open_handle(h) -> int:
    """Map a peer's (handle, offset); returns the device pointer of the peer tensor."""
    raw, off = h
    p = ctypes.c_void_p()
    _check(_lib().stokesfo_ipc_open_handle(ctypes.create_string_buffer(raw, 64), ctypes.byref(p)), "ipc_open_handle")
    return int(p.value) + off


def ipc_close(p: int):
    _check(_lib().stokesfo_ipc_close(ctypes.c_void_p(p)), "ipc_close")


# ---------------------------------------------------------------------------
# Host-side mesh construction (numpy in, numpy out)
# ---------------------------------------------------------------------------

def mesh_extrude(xy, polys, b, H, L: int):
    xy = np.ascontiguousarray(xy, dtype=np.float64)
    polys = np.ascontiguousarray(polys, dtype=np.int32)
    b = np.ascontiguousarray(b, dtype=np.float64)
    H = np.ascontiguousarray(H, dtype=np.float64)
    nv, nf, npoly = xy.shape[0], polys.shape[0], polys.shape[1]
    conn = np.empty((nf * L, 2 * npoly), dtype=np.int32)
    coords = np.empty((nv * (L + 1), 3), dtype=np.float64)
    _check(_lib().stokesfo_mesh_extrude(npoly, nv, _ptr(xy), nf, _ptr(polys), _ptr(b), _ptr(H), L,
                                        _ptr(conn), _ptr(coords)), "mesh_extrude")
    return conn, coords


def mesh_lateral_faces(polys, L: int):
    """(cell, side) of every lateral face over the footprint boundary, ordered by (f, side, layer)."""
    polys = np.ascontiguousarray(polys, dtype=np.int32)
    nf, npoly = polys.shape
    n = ctypes.c_int64(0)
    _check(_lib().stokesfo_mesh_lateral_faces(npoly, nf, _ptr(polys), L, ctypes.byref(n), None), "mesh_lateral_faces")
    faces = np.empty((n.value, 2), dtype=np.int32)
    _check(_lib().stokesfo_mesh_lateral_faces(npoly, nf, _ptr(polys), L, ctypes.byref(n), _ptr(faces)),
           "mesh_lateral_faces")
    return faces


def mesh_partition_columns(nf: int, nparts: int):
    r = np.empty(nparts + 1, dtype=np.int64)
    _check(_lib().stokesfo_mesh_partition_columns(nf, nparts, _ptr(r)), "mesh_partition_columns")
    return r


def mesh_localize(conn_part):
    conn_part = np.ascontiguousarray(conn_part, dtype=np.int32)
    nc, npc = conn_part.shape
    n = ctypes.c_int64(0)
    _check(_lib().stokesfo_mesh_localize(npc, nc, _ptr(conn_part), ctypes.byref(n), None, None), "mesh_localize")
    gids = np.empty(n.value, dtype=np.int64)
    lconn = np.empty_like(conn_part)
    _check(_lib().stokesfo_mesh_localize(npc, nc, _ptr(conn_part), ctypes.byref(n), _ptr(gids), _ptr(lconn)),
           "mesh_localize")
    return lconn, gids


def mesh_halo_list(gids_mine, gids_other):
    gids_mine = np.ascontiguousarray(gids_mine, dtype=np.int64)
    gids_other = np.ascontiguousarray(gids_other, dtype=np.int64)
    n = ctypes.c_int64(0)
    _check(_lib().stokesfo_mesh_halo_list(gids_mine.size, _ptr(gids_mine), gids_other.size, _ptr(gids_other),
                                          ctypes.byref(n), None), "mesh_halo_list")
    idx = np.empty(n.value, dtype=np.int32)
    _check(_lib().stokesfo_mesh_halo_list(gids_mine.size, _ptr(gids_mine), gids_other.size, _ptr(gids_other),
                                          ctypes.byref(n), _ptr(idx)), "mesh_halo_list")
    return idx
