"""Host logic of the generic-face TMA kernel's shared-memory staging
(csrc/bte_staging.h, used by bte_create): the half-warp bank-conflict cost
model, the per-cell face-slot order and the placement of a tile's halo / ghost
values.  Compiled here with g++ on its own (no CUDA), CPU only."""
import ctypes as C
import os
import subprocess

import numpy as np
import pytest

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(os.path.dirname(HERE), "paper_conf_ipps_heislersdms24_b200", "csrc")

HARNESS = r"""
#include "bte_staging.h"
using namespace bte_host;
extern "C" int wave16(const uint16_t *v, int n) {  // one half-warp, one slot
    uint16_t col[1][16];
    for (int i = 0; i < n; ++i) col[0][i] = v[i];
    int w, s;
    half_costs(col, 1, n, &w, &s);
    return w;
}
extern "C" void order(uint16_t *sidx, int nc, int mf, uint8_t *perm, long long *before, long long *after) {
    std::vector<uint16_t> v(sidx, sidx + (size_t)nc * mf);
    std::vector<uint8_t> p;
    auto r = order_face_slots(v, nc, mf, p);
    std::copy(v.begin(), v.end(), sidx);
    std::copy(p.begin(), p.end(), perm);
    *before = r.first;
    *after = r.second;
}
// items k = 0..n-1 read by half-warps rd[off[k] .. off[k+1]); deg[16][16] in/out
extern "C" void place(const int *off, const int *rd, int n, int *deg, int base, int cap, int *pos) {
    std::vector<std::vector<int32_t>> readers(n);
    for (int k = 0; k < n; ++k) readers[k].assign(rd + off[k], rd + off[k + 1]);
    std::vector<int32_t> out;
    place_staged(readers, reinterpret_cast<int (*)[16]>(deg), base, cap, out);
    std::copy(out.begin(), out.end(), pos);
}
"""


@pytest.fixture(scope="module")
def lib(tmp_path_factory):
    d = tmp_path_factory.mktemp("staging")
    src, so = d / "h.cpp", d / "libh.so"
    src.write_text(HARNESS)
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-I", CSRC, str(src), "-o", str(so)])
    L = C.CDLL(str(so))
    L.wave16.restype = C.c_int
    return L


def _u16(a):
    return np.ascontiguousarray(a, np.uint16)


def test_wavefront_model(lib):
    """A half-warp's 64-bit load: distinct values sharing a bank pair (index mod
    16) serialize, equal values broadcast (the rule ncu confirmed on C3t)."""
    w = lambda v: lib.wave16(_u16(v).ctypes.data_as(C.c_void_p), len(v))
    assert w(range(16)) == 1                       # 16 classes, one each
    assert w(range(100, 116)) == 1                 # (any 16 consecutive indices)
    assert w([5] * 16) == 1                        # one value: broadcast
    assert w([0, 16] + list(range(1, 15))) == 2    # 0 and 16 share bank pair 0
    assert w([0, 16, 32, 48] * 4) == 4             # four distinct values, one class
    assert w([3 + 16 * k for k in range(16)]) == 16


def _order(lib, sidx):
    mf, nc = sidx.shape
    s = _u16(sidx).copy()
    perm = np.zeros(nc * mf, np.uint8)
    b, a = C.c_longlong(), C.c_longlong()
    lib.order(s.ctypes.data_as(C.c_void_p), nc, mf, perm.ctypes.data_as(C.c_void_p), C.byref(b), C.byref(a))
    return s, perm.reshape(nc, mf), b.value, a.value


def test_face_slot_order_is_a_per_cell_permutation(lib):
    rng = np.random.default_rng(7)
    mf, nc = 3, 1000
    sidx = rng.integers(0, 384, size=(mf, nc))
    s, perm, before, after = _order(lib, sidx)
    for c in range(nc):
        assert sorted(perm[c]) == list(range(mf))
        assert list(s[:, c]) == [sidx[perm[c][j], c] for j in range(mf)]
    assert after <= before
    s2, perm2, _, after2 = _order(lib, sidx)  # deterministic
    assert np.array_equal(s, s2) and after2 == after


def test_face_slot_order_on_a_triangle_mesh(lib):
    """C6t's triangles in tiles of 256 consecutive cells (own index = cell - tile
    start, out-of-tile neighbours after 256): the order removes a large share of
    the conflicts; the cost never exceeds the caller's order."""
    from paper_conf_ipps_heislersdms24_b200 import inputs as gen
    m = gen.make_config("C6t").mesh
    nc, off, nbr = m["n_cells"], m["face_offsets"], m["face_nbr"]
    sidx = np.zeros((3, nc), np.int64)
    for t0 in range(0, nc, 256):
        halo = {}
        for c in range(t0, min(nc, t0 + 256)):
            for j, f in enumerate(range(off[c], off[c + 1])):
                v = nbr[f]
                if t0 <= v < t0 + 256:
                    sidx[j, c] = v - t0
                else:
                    sidx[j, c] = 256 + halo.setdefault(int(v), len(halo))
    _, _, before, after = _order(lib, sidx)
    assert after <= 0.8 * before, (before, after)


def test_placement_spreads_bank_classes(lib):
    """Items read by a half-warp whose in-tile reads crowd some bank classes
    land on the free classes; positions are distinct and inside the window."""
    n, base, cap = 12, 256, 128
    deg = np.zeros((16, 16), np.int32)
    deg[0, :8] = 3  # half-warp 0 already reads classes 0..7 three times
    off = np.arange(n + 1, dtype=np.int32)
    rd = np.zeros(n, np.int32)  # every item read by half-warp 0
    pos = np.zeros(n, np.int32)
    lib.place(off.ctypes.data_as(C.c_void_p), rd.ctypes.data_as(C.c_void_p), n, deg.ctypes.data_as(C.c_void_p),
              base, cap, pos.ctypes.data_as(C.c_void_p))
    assert len(set(pos)) == n and pos.min() >= base and pos.max() < base + cap
    cls = pos & 15
    assert set(cls[:8]) == set(range(8, 16))  # the 8 empty classes first
    assert cls.min() >= 8                      # never onto the crowded classes
    assert list(deg[0]) == [3] * 8 + [2] * 4 + [1] * 4
