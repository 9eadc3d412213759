"""CPU-side checks of the product library: it loads, exports every symbol
include/stokesfo.h declares, and its host mesh construction (extrusion,
partition, localisation, halo lists) is bit-exact with the oracle's
independent set-algebra versions."""
import ctypes
import os
import re

import numpy as np
import pytest

import oracle as O
from paper_conf_sc_antepara0cw24_b200 import stokesfo as S
from paper_conf_sc_antepara0cw24_b200 import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_library_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "stokesfo.h")).read()
    declared = set(re.findall(r"\b(stokesfo_[a-z_]+)\s*\(", hdr))
    assert len(declared) >= 18
    lib = ctypes.CDLL(S.lib_path() if os.path.exists(S.lib_path()) else S._build.build())
    for name in sorted(declared):
        assert hasattr(lib, name), name
    assert declared == set(S.EXPORTS)


def test_library_is_sm100a():
    import subprocess
    path = S._build.build()
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", path], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_strerror_and_create_validation_without_gpu():
    lib = S._lib()
    assert lib.stokesfo_strerror(5).decode().startswith("unsupported")
    d = S.Desc()
    d.abi_version = 1
    d.elem = 0
    d.num_cells = 10
    n = ctypes.c_size_t()
    assert lib.stokesfo_workspace_size(ctypes.byref(d), ctypes.byref(n)) == 0
    assert n.value == 256 + 3 * 6560   # header + three hex8 records of 4 cells (10 cells)
    d.glen_n = 2.0
    d.delta = 1e-10
    h = ctypes.c_void_p()
    # missing conn/coords -> EINVAL before any CUDA call
    assert lib.stokesfo_create(ctypes.byref(d), ctypes.byref(h)) == 1


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_extrusion_bit_exact_vs_oracle(elem):
    fp = synth.tiny_footprint(jitter=0.2, seed=7)
    if elem == "wedge6":
        fp = synth.split_to_triangles(fp)
    for L in (1, 5):
        c1, x1 = S.mesh_extrude(fp.xy, fp.polys, fp.b, fp.H, L)
        c2, x2 = O.extrude(fp.xy, fp.polys, fp.b, fp.H, L)
        assert np.array_equal(c1, c2)
        assert np.array_equal(x1.view(np.int64), x2.view(np.int64))   # bit-exact coordinates


def test_extrusion_antarctica_counts():
    fp = synth.antarctica_footprint()
    conn, coords = S.mesh_extrude(fp.xy, fp.polys, fp.b, fp.H, 10)
    assert conn.shape == (8431650, 8) and coords.shape == (9313304, 3)
    c2, x2 = O.extrude(fp.xy, fp.polys, fp.b, fp.H, 10)
    assert np.array_equal(conn, c2)
    assert np.array_equal(coords.view(np.int64), x2.view(np.int64))


@pytest.mark.parametrize("P", [1, 2, 3, 8])
def test_partition_localize_halo_bit_exact(P):
    fp = synth.tiny_footprint(n=8, jitter=0.1, seed=2)
    L = 3
    conn, coords = O.extrude(fp.xy, fp.polys, fp.b, fp.H, L)
    r1 = S.mesh_partition_columns(fp.nf, P)
    r2 = O.partition_columns(fp.nf, P)
    assert np.array_equal(r1, r2)
    parts = []
    for r in range(P):
        lc, g = S.mesh_localize(conn[r1[r] * L:r1[r + 1] * L])
        lc2, g2 = O.local_mesh(conn, L, r2[r], r2[r + 1])
        assert np.array_equal(lc, lc2) and np.array_equal(g, g2)
        parts.append(g)
    halo = O.halo_lists(parts)
    for r in range(P):
        for s in range(P):
            if r == s:
                continue
            idx = S.mesh_halo_list(parts[r], parts[s])
            if (r, s) in halo:
                assert np.array_equal(idx, halo[(r, s)])
            else:
                assert idx.size == 0


def test_create_rejects_bad_descriptors_without_gpu():
    """Validation happens before any CUDA call: sizes beyond int32 node ids, negative
    counts, bad element/geometry modes, wrong ABI version, non-positive delta."""
    lib = S._lib()

    def desc(**kw):
        d = S.Desc()
        d.abi_version, d.elem, d.num_cells, d.num_nodes = 1, 0, 4, 10
        d.conn, d.coords = ctypes.c_void_p(256), ctypes.c_void_p(512)
        d.glen_n, d.delta, d.k = 3.0, 1e-10, 1.0
        d.workspace, d.workspace_bytes = ctypes.c_void_p(1024), 1 << 20
        for k, v in kw.items():
            setattr(d, k, v)
        return d

    h = ctypes.c_void_p()
    for bad, code in ((dict(num_nodes=2 ** 31), 1), (dict(num_cells=-1), 1), (dict(elem=7), 1),
                      (dict(abi_version=2), 1), (dict(delta=0.0), 1), (dict(glen_n=4.0), 5),
                      (dict(geometry_mode=3), 1), (dict(workspace=ctypes.c_void_p(1032)), 1),
                      (dict(coords=ctypes.c_void_p(520)), 1), (dict(workspace_bytes=100), 4)):
        assert lib.stokesfo_create(ctypes.byref(desc(**bad)), ctypes.byref(h)) == code, bad
    n = ctypes.c_size_t()
    assert lib.stokesfo_workspace_size(ctypes.byref(desc(geometry_mode=1)), ctypes.byref(n)) == 0
    assert n.value == 256 + ((10 * 32 + 255) // 256) * 256      # header + double4 coordinates


@pytest.mark.parametrize("elem", ["hex8", "wedge6"])
def test_lateral_faces_bit_exact_vs_oracle(elem):
    """NEXT-4 (reading Z19): the library's boundary-side set equals the oracle's set algebra."""
    from oracle import lateral as LT
    fp = synth.tiny_footprint(n=7, jitter=0.2, seed=4)
    if elem == "wedge6":
        fp = synth.split_to_triangles(fp)
    for L in (1, 4):
        got = S.mesh_lateral_faces(fp.polys, L)
        assert np.array_equal(got, LT.lateral_faces(fp.polys, L))


def test_lateral_faces_antarctica_vs_oracle():
    """C4 footprint (ragged, masked margin with embayments): same set, bit-exact."""
    from oracle import lateral as LT
    fp = synth.antarctica_footprint(h=16.0)
    got = S.mesh_lateral_faces(fp.polys, 2)
    assert got.shape[0] > 0
    assert np.array_equal(got, LT.lateral_faces(fp.polys, 2))
