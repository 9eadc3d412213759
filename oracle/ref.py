"""Python side of the oracle (TEST INFRASTRUCTURE ONLY -- see oracle/__init__.py).

* ctypes wrapper of ``oracle.c`` (built with plain gcc on first use);
* O1 extrusion and numbering, numpy;
* O9 CSR pattern, column partition and halo lists as plain set algebra;
* a numpy complex-capable residual (eq. (1) weak form, Fig. 2),
  used for complex-step derivatives: an independent pin of the C AD Jacobian.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(HERE, "oracle.c")
_LIB = os.path.join(HERE, "liboracle.so")

HEX8, WEDGE6 = 0, 1
ELEM = {"hex8": HEX8, "wedge6": WEDGE6}
NODES = {HEX8: 8, WEDGE6: 6}
QPS = {HEX8: 8, WEDGE6: 6}


def build_oracle(force: bool = False) -> str:
    """Compile oracle.c with plain gcc (-O2 -fopenmp); returns the .so path."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build_oracle())
        P = ctypes.c_void_p
        I64 = ctypes.c_int64
        D = ctypes.c_double
        _lib.oracle_geometry.argtypes = [ctypes.c_int, I64, P, P, P, P]
        _lib.oracle_geometry.restype = I64
        _lib.oracle_eval.argtypes = [ctypes.c_int, I64, P, P, P, P, P, P, P, D, D, D, D,
                                     ctypes.c_int, P, P, P]
        _lib.oracle_eval.restype = None
        _lib.oracle_gather.argtypes = [ctypes.c_int, I64, P, P, P]
        _lib.oracle_scatter.argtypes = [ctypes.c_int, I64, P, P, P]
        _lib.oracle_scatter_csr.argtypes = [ctypes.c_int, I64, P, P, P, P, P]
        _lib.oracle_scatter_csr.restype = I64
        _lib.oracle_ref_element.argtypes = [ctypes.c_int, P, P, P]
        _lib.oracle_basis_at.argtypes = [ctypes.c_int, P, P, P]
        _lib.oracle_quadrature.argtypes = [ctypes.c_int, P, P]
        _lib.oracle_num_threads.restype = ctypes.c_int
        _lib.oracle_set_num_threads.argtypes = [ctypes.c_int]
        _lib.oracle_set_num_threads.restype = None
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _c(a, dtype):
    return None if a is None else np.ascontiguousarray(a, dtype=dtype)


def num_threads() -> int:
    return int(lib().oracle_num_threads())


def set_num_threads(n: int) -> None:
    """OpenMP threads of the oracle's cell loops (timing only; results do not depend on it)."""
    lib().oracle_set_num_threads(int(n))


# ---------------------------------------------------------------------------
# O2 reference element
# ---------------------------------------------------------------------------

def ref_element(elem: int):
    """(BF[N][Q], dBF[N][Q][3], w[Q]) of the reference element (O2)."""
    N, Q = NODES[elem], QPS[elem]
    bf = np.zeros((N, Q))
    dbf = np.zeros((N, Q, 3))
    w = np.zeros(Q)
    lib().oracle_ref_element(elem, _p(bf), _p(dbf), _p(w))
    return bf, dbf, w


def quadrature(elem: int):
    Q = QPS[elem]
    xq = np.zeros((Q, 3))
    w = np.zeros(Q)
    lib().oracle_quadrature(elem, _p(xq), _p(w))
    return xq, w


def basis_at(elem: int, p):
    N = NODES[elem]
    p = np.ascontiguousarray(p, dtype=np.float64)
    phi = np.zeros(N)
    dphi = np.zeros((N, 3))
    lib().oracle_basis_at(elem, _p(p), _p(phi), _p(dphi))
    return phi, dphi


# ---------------------------------------------------------------------------
# O1 extrusion and numbering (reading Z10)
# ---------------------------------------------------------------------------

def extrude(xy, polys, b, H, L: int):
    """Extrude a footprint by L uniform-sigma layers.

    node(v,k) = v*(L+1)+k, k = 0 (bed) .. L (surface);
    cell(f,k) = f*L+k;  conn = [poly at level k, poly at level k+1];
    z = b_v + H_v * (k/L)   (k/L evaluated first, in fp64).
    Returns (conn [C][2*npoly] int32, coords [nodes][3] fp64).
    """
    xy = np.asarray(xy, dtype=np.float64)
    polys = np.asarray(polys, dtype=np.int64)
    nv, npoly = xy.shape[0], polys.shape[1]
    nf = polys.shape[0]
    k = np.arange(L + 1)
    t = k.astype(np.float64) / float(L)
    coords = np.empty((nv, L + 1, 3))
    coords[:, :, 0] = xy[:, 0:1]
    coords[:, :, 1] = xy[:, 1:2]
    coords[:, :, 2] = np.asarray(b)[:, None] + np.asarray(H)[:, None] * t[None, :]
    kk = np.arange(L)
    bot = polys[:, None, :] * (L + 1) + kk[None, :, None]          # [nf][L][npoly]
    conn = np.concatenate([bot, bot + 1], axis=2).reshape(nf * L, 2 * npoly)
    return conn.astype(np.int32), coords.reshape(nv * (L + 1), 3)


# ---------------------------------------------------------------------------
# O3 geometry, O4-O7 evaluation, O8 scatter (ctypes into oracle.c)
# ---------------------------------------------------------------------------

def geometry(elem: int, conn, coords):
    """(GradBF[C][N][Q][3], wMeasure[C][Q], n_bad) -- O3."""
    conn = _c(conn, np.int32)
    coords = _c(coords, np.float64)
    C = conn.shape[0]
    N, Q = NODES[elem], QPS[elem]
    G = np.zeros((C, N, Q, 3))
    wm = np.zeros((C, Q))
    bad = lib().oracle_geometry(elem, C, _p(conn), _p(coords), _p(G), _p(wm))
    return G, wm, int(bad)


def evaluate(elem: int, conn, G, wm, U, surface=None, force_qp=None, kc=None,
             k=10.77, glen_n=3.0, delta=1e-10, rho_g=8.927, mode: str = "resid"):
    """Element evaluation (O4-O7).

    mode: "resid" (Fig. 2 optimized order), "jac" (forward-AD, residual too),
    "resid_baseline" (Fig. 2 baseline order), "jac_analytic" (closed form).
    Returns dict with mu_qp [C][Q], R_cell [C][N][2], J_cell [C][2N][2N].
    """
    m = {"resid": 0, "jac": 1, "resid_baseline": 2, "jac_analytic": 3}[mode]
    conn = _c(conn, np.int32)
    G = _c(G, np.float64)
    wm = _c(wm, np.float64)
    U = _c(U, np.float64)
    surface = _c(surface, np.float64)
    force_qp = _c(force_qp, np.float64)
    kc = _c(kc, np.float64)
    C = conn.shape[0]
    N, Q = NODES[elem], QPS[elem]
    mu = np.zeros((C, Q)) if m in (0, 1) else None
    R = np.zeros((C, N, 2)) if m != 3 else None
    J = np.zeros((C, 2 * N, 2 * N)) if m in (1, 3) else None
    lib().oracle_eval(elem, C, _p(conn), _p(G), _p(wm), _p(U), _p(surface), _p(force_qp),
                      _p(kc), k, glen_n, delta, rho_g, m, _p(mu), _p(R), _p(J))
    return {"mu_qp": mu, "R_cell": R, "J_cell": J}


def gather(elem: int, conn, U):
    conn = _c(conn, np.int32)
    U = _c(U, np.float64)
    out = np.zeros((conn.shape[0], NODES[elem], 2))
    lib().oracle_gather(elem, conn.shape[0], _p(conn), _p(U), _p(out))
    return out


def scatter(elem: int, conn, R_cell, num_nodes: int, R=None):
    conn = _c(conn, np.int32)
    R_cell = _c(R_cell, np.float64)
    R = np.zeros((num_nodes, 2)) if R is None else np.ascontiguousarray(R, dtype=np.float64).copy()
    lib().oracle_scatter(elem, conn.shape[0], _p(conn), _p(R_cell), _p(R))
    return R


def scatter_csr(elem: int, conn, J_cell, rowptr, colidx, vals=None):
    conn = _c(conn, np.int32)
    J_cell = _c(J_cell, np.float64)
    rowptr = _c(rowptr, np.int64)
    colidx = _c(colidx, np.int32)
    vals = np.zeros(colidx.shape[0]) if vals is None else np.ascontiguousarray(vals, dtype=np.float64).copy()
    miss = lib().oracle_scatter_csr(elem, conn.shape[0], _p(conn), _p(J_cell), _p(rowptr),
                                    _p(colidx), _p(vals))
    return vals, int(miss)


# ---------------------------------------------------------------------------
# O9 CSR pattern, partition and halo lists: plain set algebra
# ---------------------------------------------------------------------------

def csr_pattern(conn, num_nodes: int):
    """Rows = dofs 2*node+comp; columns = sorted set of dofs sharing a cell."""
    conn = np.asarray(conn)
    nbrs = [set() for _ in range(num_nodes)]
    for c in range(conn.shape[0]):
        cell = [int(x) for x in conn[c]]
        for i in cell:
            nbrs[i].update(cell)
    rowptr = [0]
    colidx = []
    for node in range(num_nodes):
        cols = sorted(nbrs[node])
        for a in range(2):
            for j in cols:
                colidx.extend((2 * j, 2 * j + 1))
            rowptr.append(len(colidx))
    return np.array(rowptr, dtype=np.int64), np.array(colidx, dtype=np.int32)


def partition_columns(nf: int, nparts: int):
    """Column ranges: part r owns footprint columns [r*nf//P, (r+1)*nf//P)."""
    return np.array([(r * nf) // nparts for r in range(nparts + 1)], dtype=np.int64)


def local_mesh(conn, L: int, col_lo: int, col_hi: int):
    """Cells of columns [col_lo, col_hi): local node ids = rank of the global id
    among the sorted set of touched global nodes.  Returns
    (local_conn, global_node_ids)."""
    cells = conn[col_lo * L:col_hi * L]
    gids = np.array(sorted(set(int(x) for x in cells.reshape(-1))), dtype=np.int64)
    lut = {g: i for i, g in enumerate(gids)}
    lconn = np.array([[lut[int(x)] for x in row] for row in cells], dtype=np.int32).reshape(cells.shape)
    return lconn, gids


def halo_lists(gid_sets):
    """For every ordered pair (r, s), r != s, the local ids on r of the global
    nodes r shares with s, ordered by global id."""
    out = {}
    for r, gr in enumerate(gid_sets):
        pos = {int(g): i for i, g in enumerate(gr)}
        for s, gs in enumerate(gid_sets):
            if s == r:
                continue
            shared = sorted(set(int(g) for g in gr) & set(int(g) for g in gs))
            if shared:
                out[(r, s)] = np.array([pos[g] for g in shared], dtype=np.int32)
    return out


# ---------------------------------------------------------------------------
# numpy complex-capable residual (independent of oracle.c) for complex step
# ---------------------------------------------------------------------------

def resid_numpy(elem: int, G, wm, Uc, sc, kc, glen_n=3.0, delta=1e-10, rho_g=8.927, bf=None):
    """R[c][n][a] = sum_q wM (sigma_(a,.) . GradBF[n][q] + f_a BF[n][q]) with
    sigma from Fig. 2, f = rho g grad s_h (eq. (1)).  Uc may be
    complex (complex step).  bf = BF[N][Q] table (from the oracle's O2)."""
    p = (1.0 - glen_n) / (2.0 * glen_n)
    ug = np.einsum("cna,cnqd->cqad", Uc, G)
    ux, uy, uz = ug[..., 0, 0], ug[..., 0, 1], ug[..., 0, 2]
    vx, vy, vz = ug[..., 1, 0], ug[..., 1, 1], ug[..., 1, 2]
    e2 = ux * ux + vy * vy + ux * vy + 0.25 * (uy + vx) ** 2 + 0.25 * uz * uz + 0.25 * vz * vz
    mu = np.asarray(kc)[:, None] * (e2 + delta) ** p
    s00 = 2 * mu * (2 * ux + vy)
    s11 = 2 * mu * (2 * vy + ux)
    s01 = mu * (uy + vx)
    s02 = mu * uz
    s12 = mu * vz
    wg = G * wm[:, None, :, None]
    R0 = np.einsum("cq,cnq->cn", s00, wg[..., 0]) + np.einsum("cq,cnq->cn", s01, wg[..., 1]) \
        + np.einsum("cq,cnq->cn", s02, wg[..., 2])
    R1 = np.einsum("cq,cnq->cn", s01, wg[..., 0]) + np.einsum("cq,cnq->cn", s11, wg[..., 1]) \
        + np.einsum("cq,cnq->cn", s12, wg[..., 2])
    if sc is not None:
        gs = np.einsum("cn,cnqd->cqd", sc, G[..., 0:2])
        wbf = bf[None, :, :] * wm[:, None, :]
        R0 = R0 + np.einsum("cq,cnq->cn", rho_g * gs[..., 0], wbf)
        R1 = R1 + np.einsum("cq,cnq->cn", rho_g * gs[..., 1], wbf)
    return np.stack([R0, R1], axis=-1)


def jac_complex_step(elem: int, G, wm, Uc, sc, kc, h=1e-30, **kw):
    """J[c][k][l] = Im R_k(U + i h e_l) / h, l = 2n+b (complex step)."""
    C, N = Uc.shape[0], Uc.shape[1]
    nd = 2 * N
    J = np.zeros((C, nd, nd))
    for l in range(nd):
        Up = Uc.astype(np.complex128)
        Up[:, l // 2, l % 2] += 1j * h
        R = resid_numpy(elem, G, wm, Up, sc, kc, **kw)
        J[:, :, l] = R.reshape(C, nd).imag / h
    return J


def jac_central_fd(elem: int, G, wm, Uc, sc, kc, rel=1e-6, **kw):
    """Central finite differences of the numpy residual, h = rel*max|U|."""
    C, N = Uc.shape[0], Uc.shape[1]
    nd = 2 * N
    J = np.zeros((C, nd, nd))
    scale = np.maximum(np.abs(Uc).reshape(C, -1).max(axis=1), 1.0)
    for l in range(nd):
        hh = rel * scale
        Up = Uc.copy()
        Um = Uc.copy()
        Up[:, l // 2, l % 2] += hh
        Um[:, l // 2, l % 2] -= hh
        Rp = resid_numpy(elem, G, wm, Up, sc, kc, **kw).reshape(C, nd)
        Rm = resid_numpy(elem, G, wm, Um, sc, kc, **kw).reshape(C, nd)
        J[:, :, l] = (Rp - Rm) / (2 * hh[:, None])
    return J
