"""TEST INFRASTRUCTURE -- Python face of the fp64 CPU oracle (bvh_oracle.cpp).

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
``--impl reference``) may import this module.  It shares no code with the
CUDA path.  Citations: P:NNN = line of /root/reference/PAPER.md; [A#] =
reading in DESIGN.md.

``step()`` composes Alg. 6 from the C++ pieces:
bbox -> keys -> stable sort -> permute -> build -> force -> leapfrog (O8).

``precision=32`` (default): fp32 bodies, the state precision of the path
under test.  ``precision=64`` (NEXT-2): fp64 bodies and state -- the paper's
own precision throughout; every stage evaluates the same
expressions on the doubles.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import time
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "bvh_oracle.cpp")
_LIB = os.path.join(_HERE, "libbvh_oracle.so")
_lib = None

_P = C.c_void_p
_f32p = np.ctypeslib.ndpointer(np.float32, flags="C_CONTIGUOUS")
_f64p = np.ctypeslib.ndpointer(np.float64, flags="C_CONTIGUOUS")
_u32p = np.ctypeslib.ndpointer(np.uint32, flags="C_CONTIGUOUS")
_u64p = np.ctypeslib.ndpointer(np.uint64, flags="C_CONTIGUOUS")
_i64p = np.ctypeslib.ndpointer(np.int64, flags="C_CONTIGUOUS")


def build(force: bool = False) -> str:
    """Compile the oracle (plain g++, no fast-math, no contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = f"{_LIB}.{os.getpid()}.tmp"  # concurrent builders (multi-rank tests) never share a temp file
        cmd = ["g++", "-O2", "-std=c++17", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
               "-pthread", "-o", tmp, _SRC]
        subprocess.run(cmd, check=True)
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        L.orc_paper_key_bits.argtypes = [C.c_int64]
        L.orc_paper_key_bits.restype = C.c_int
        L.orc_hilbert_index.argtypes = [C.c_uint32, C.c_uint32, C.c_uint32, C.c_int]
        L.orc_hilbert_index.restype = C.c_uint64
        L.orc_bbox.argtypes = [C.c_int64, _f32p, _f32p, _f32p]
        L.orc_quantize.argtypes = [C.c_int64, _f32p, _f32p, _f32p, C.c_int, _u32p]
        L.orc_keys.argtypes = [C.c_int64, _f32p, C.c_int, _u64p]
        L.orc_sort.argtypes = [C.c_int64, _u64p, _u32p]
        L.orc_build.argtypes = [C.c_int64, _f32p, _f32p]
        L.orc_build.restype = _P
        L.orc_free_tree.argtypes = [_P]
        L.orc_free_tree.restype = None
        L.orc_tree_levels.argtypes = [_P]
        L.orc_tree_count.argtypes = [_P, C.c_int]
        L.orc_tree_count.restype = C.c_int64
        L.orc_tree_level.argtypes = [_P, C.c_int, _P, _P, _P, _P, _P]
        L.orc_force.argtypes = [_P, C.c_double, C.c_double, _i64p, C.c_int64, _f64p, _P, C.c_int]
        L.orc_force_q.argtypes = [_P, C.c_double, C.c_double, C.c_int, _i64p, C.c_int64, _f64p, _P, C.c_int]
        L.orc_force_q.restype = C.c_int
        L.orc_tree_level_quad.argtypes = [_P, C.c_int, _f64p]
        L.orc_tree_level_quad.restype = C.c_int
        L.orc_force_list.argtypes = [_P, C.c_double, C.c_double, C.c_int64, _i64p, C.c_int64]
        L.orc_force_list.restype = C.c_int64
        L.orc_direct.argtypes = [C.c_int64, _f32p, _f32p, C.c_double, _i64p, C.c_int64, _f64p, C.c_int]
        L.orc_bbox_d.argtypes = [C.c_int64, _f64p, _f64p, _f64p]
        L.orc_quantize_d.argtypes = [C.c_int64, _f64p, _f64p, _f64p, C.c_int, _u32p]
        L.orc_keys_d.argtypes = [C.c_int64, _f64p, C.c_int, _u64p]
        L.orc_build_d.argtypes = [C.c_int64, _f64p, _f64p]
        L.orc_build_d.restype = _P
        L.orc_tree_level_box_d.argtypes = [_P, C.c_int, _f64p, _f64p]
        L.orc_direct_d.argtypes = [C.c_int64, _f64p, _f64p, C.c_double, _i64p, C.c_int64, _f64p, C.c_int]
        for f in ("orc_bbox", "orc_quantize", "orc_keys", "orc_sort", "orc_tree_levels", "orc_tree_level",
                  "orc_force", "orc_direct", "orc_bbox_d", "orc_quantize_d", "orc_keys_d", "orc_tree_level_box_d",
                  "orc_direct_d"):
            getattr(L, f).restype = C.c_int
        _lib = L
    return _lib


def _ok(rc: int, what: str):
    if rc != 0:
        raise ValueError(f"oracle {what} failed (rc={rc})")


def _f32(a, shape=None):
    a = np.ascontiguousarray(a, np.float32)
    if shape is not None:
        a = a.reshape(shape)
    return a


def _real(a, precision, shape=None):
    """fp32 or fp64 contiguous array for the given precision (32 or 64)."""
    if precision not in (32, 64):
        raise ValueError("precision must be 32 or 64")
    a = np.ascontiguousarray(a, np.float32 if precision == 32 else np.float64)
    if shape is not None:
        a = a.reshape(shape)
    return a


# ------------------------------------------------------------------ O1..O4 --
def paper_key_bits(n: int) -> int:
    """[A8] smallest b >= 1 with 8^b >= N."""
    return lib().orc_paper_key_bits(int(n))


def resolve_key_bits(n: int, key_bits: int) -> int:
    return paper_key_bits(n) if key_bits == 0 else int(key_bits)


def hilbert_index(x: int, y: int, z: int, b: int) -> int:
    """Skilling's transpose + MSB-first interleave (ref [17])."""
    return int(lib().orc_hilbert_index(x, y, z, b))


def bbox(pos, precision: int = 32):
    """O1 -- Alg. 3."""
    pos = _real(pos, precision, (-1, 3))
    lo = np.empty(3, pos.dtype)
    hi = np.empty(3, pos.dtype)
    f = lib().orc_bbox if precision == 32 else lib().orc_bbox_d
    _ok(f(len(pos), pos, lo, hi), "bbox")
    return lo, hi


def quantize(pos, b: int, precision: int = 32):
    """O2 -- grid cells [A9][A17]."""
    pos = _real(pos, precision, (-1, 3))
    lo, hi = bbox(pos, precision)
    q = np.empty((len(pos), 3), np.uint32)
    f = lib().orc_quantize if precision == 32 else lib().orc_quantize_d
    _ok(f(len(pos), pos, lo, hi, int(b), q), "quantize")
    return q


def keys(pos, b: int, precision: int = 32):
    """O1..O3 -- Hilbert key per body in current slot order."""
    pos = _real(pos, precision, (-1, 3))
    out = np.empty(len(pos), np.uint64)
    f = lib().orc_keys if precision == 32 else lib().orc_keys_d
    _ok(f(len(pos), pos, int(b), out), "keys")
    return out


def sort_perm(k):
    """O4 -- stable sort; perm[k] = current slot of the body now at slot k."""
    k = np.ascontiguousarray(k, np.uint64)
    perm = np.empty(len(k), np.uint32)
    _ok(lib().orc_sort(len(k), k, perm), "sort")
    return perm


# --------------------------------------------------------------------- O6 --
@dataclass
class LevelData:
    M: np.ndarray      # fp64 [c]
    com: np.ndarray    # fp64 [c,3]
    s2: np.ndarray     # fp64 [c]
    lo: np.ndarray     # fp32 [c,3] (fp64 for a precision-64 tree)
    hi: np.ndarray     # fp32 [c,3] (fp64 for a precision-64 tree)

    @property
    def m32(self):
        return self.M.astype(np.float32)

    @property
    def c32(self):
        return self.com.astype(np.float32)


class Tree:
    """O6 -- BUILDTREEACCUMULATEMASS over Hilbert-sorted bodies."""

    def __init__(self, pos_sorted, mass_sorted, precision: int = 32):
        self.precision = precision
        self.pos = _real(pos_sorted, precision, (-1, 3))
        self.mass = _real(mass_sorted, precision, (-1,))
        if len(self.pos) != len(self.mass) or len(self.pos) < 1:
            raise ValueError("bad tree input")
        self.n = len(self.pos)
        build_fn = lib().orc_build if precision == 32 else lib().orc_build_d
        self._h = build_fn(self.n, self.pos, self.mass)
        if not self._h:
            raise MemoryError("orc_build failed")
        self.L = lib().orc_tree_levels(self._h)

    def __del__(self):
        h = getattr(self, "_h", None)
        if h and _lib is not None:
            _lib.orc_free_tree(h)
            self._h = None

    def count(self, level: int) -> int:
        return int(lib().orc_tree_count(self._h, level))

    def level(self, l: int) -> LevelData:
        c = self.count(l)
        if c < 0:
            raise IndexError(l)
        d = LevelData(np.empty(c), np.empty((c, 3)), np.empty(c), np.empty((c, 3), np.float32),
                      np.empty((c, 3), np.float32))
        _ok(lib().orc_tree_level(self._h, l, d.M.ctypes.data, d.com.ctypes.data, d.s2.ctypes.data,
                                 d.lo.ctypes.data, d.hi.ctypes.data), "tree_level")
        if self.precision == 64:
            d.lo = np.empty((c, 3))
            d.hi = np.empty((c, 3))
            _ok(lib().orc_tree_level_box_d(self._h, l, d.lo, d.hi), "tree_level_box_d")
        return d

    def force(self, theta: float, eps: float, targets=None, nthreads: int = 0, quad: bool = False):
        """O7 -- per-target DFS; returns (acc fp64 [nt,3], interactions int64 [nt]).
        ``quad`` adds the quadrupole of every accepted node (NEXT-4 [A24])."""
        t = np.arange(self.n, dtype=np.int64) if targets is None else np.ascontiguousarray(targets, np.int64)
        acc = np.empty((len(t), 3))
        cnt = np.empty(len(t), np.int64)
        _ok(lib().orc_force_q(self._h, float(theta), float(eps), int(bool(quad)), t, len(t), acc, cnt.ctypes.data,
                              int(nthreads)), "force")
        return acc, cnt

    def level_quad(self, l: int):
        """[A24] second moments about the COM of level l: fp64 [c, 6] (xx, yy, zz, xy, xz, yz)."""
        out = np.empty((self.count(l), 6))
        _ok(lib().orc_tree_level_quad(self._h, l, out), "tree_level_quad")
        return out

    def force_list(self, theta: float, eps: float, target: int):
        """O7 interaction list of one target: int64 [len, 2] of (level, index), DFS order."""
        cap = 4 * self.n + 64
        out = np.empty(2 * cap, np.int64)
        c = lib().orc_force_list(self._h, float(theta), float(eps), int(target), out, cap)
        if c < 0:
            raise ValueError("force_list failed")
        return out[: 2 * c].reshape(c, 2)


def direct(pos, mass, eps: float, targets=None, nthreads: int = 0, precision: int = 32):
    """D -- direct summation of Eq. 1, softened, fp64 arithmetic on
    fp32 (precision=32) or fp64 (precision=64) bodies."""
    pos = _real(pos, precision, (-1, 3))
    mass = _real(mass, precision, (-1,))
    t = np.arange(len(pos), dtype=np.int64) if targets is None else np.ascontiguousarray(targets, np.int64)
    acc = np.empty((len(t), 3))
    f = lib().orc_direct if precision == 32 else lib().orc_direct_d
    _ok(f(len(pos), pos, mass, float(eps), t, len(t), acc, int(nthreads)), "direct")
    return acc


# ------------------------------------------------------------- the step ---
@dataclass
class StepResult:
    keys: np.ndarray        # u64 [n], pre-sort slot order
    perm: np.ndarray        # u32 [n]: sorted slot k <- previous slot perm[k]
    tree: Tree
    acc: np.ndarray         # fp64 [nt,3] for `targets` (sorted slots)
    count: np.ndarray       # int64 [nt]
    targets: np.ndarray     # sorted slots the force was evaluated for
    pos: np.ndarray         # fp32 [n,3] sorted, after the update (if integrated); fp64 at precision 64
    vel: np.ndarray         # fp32 [n,3] sorted, after the update; fp64 at precision 64
    mass: np.ndarray        # fp32 [n] sorted; fp64 at precision 64
    ids: np.ndarray         # int64 [n]: body id in each sorted slot
    seconds: float


def step(pos, vel, mass, ids=None, *, theta: float, eps: float, dt: float, key_bits: int = 16,
         integrate: bool = True, targets=None, nthreads: int = 0, resort: bool = True,
         quad: bool = False, precision: int = 32) -> StepResult:
    """One step of Alg. 6 on fp32 state in the current slot order.

    O8 [A14] kick-drift leapfrog, v_{+1/2} = v_{-1/2} + a dt, x += v_{+1/2} dt,
    evaluated in fp64 and stored in fp32 (the state precision of the path).
    ``precision=64`` (NEXT-2): fp64 state in, fp64 state out, every stage on
    the doubles (the paper's precision).
    With ``targets`` (sorted slots) only those bodies get forces and the
    update is skipped.

    ``resort=False`` is the tree-reuse variant (NEXT-3(iii), Iwasawa et al.
    as cited at P:320, [A23]): HILBERTSORT is skipped and the bodies keep
    their current slot order (the previous step's Hilbert order); the BVH is
    rebuilt bottom-up over that order at the current positions.
    """
    t0 = time.perf_counter()
    pos = _real(pos, precision, (-1, 3))
    vel = _real(vel, precision, (-1, 3))
    mass = _real(mass, precision, (-1,))
    n = len(pos)
    ids = np.arange(n, dtype=np.int64) if ids is None else np.asarray(ids, np.int64)
    if resort:
        b = resolve_key_bits(n, key_bits)
        k = keys(pos, b, precision)            # O1-O3
        perm = sort_perm(k)                    # O4
    else:
        k = np.zeros(0, np.uint64)
        perm = np.arange(n, dtype=np.uint32)
    ps, vs, ms, ids_s = pos[perm], vel[perm], mass[perm], ids[perm]  # O5 [A11]
    tree = Tree(ps, ms, precision)             # O6
    full = targets is None
    tg = np.arange(n, dtype=np.int64) if full else np.ascontiguousarray(targets, np.int64)
    acc, cnt = tree.force(theta, eps, tg, nthreads, quad)   # O7 (+ NEXT-4 quadrupoles)
    if integrate and full:                     # O8
        v_new = vs.astype(np.float64) + acc * dt
        x_new = ps.astype(np.float64) + v_new * dt
        vs = v_new.astype(pos.dtype)
        ps = x_new.astype(pos.dtype)
    return StepResult(k, perm, tree, acc, cnt, tg, ps, vs, ms, ids_s, time.perf_counter() - t0)
