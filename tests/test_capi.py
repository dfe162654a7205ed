"""CPU-side checks of the C-ABI library: it builds, loads, and exports every
symbol include/nbody.h declares; host-only argument validation; the
independence of the oracle and the CUDA sources.  No compute calls."""
import ctypes as C
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "nbody.h")
CSRC = os.path.join(ROOT, "paper_conf_sc_casselldahg24_b200", "csrc")


def _declared():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(nbody_[a-z_0-9]+)\s*\(", text)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_sc_casselldahg24_b200 import _capi
    return _capi.load()


def test_header_declares_the_north_star_calls():
    d = _declared()
    for name in ("nbody_create", "nbody_set_bodies", "nbody_step", "nbody_get_accel", "nbody_get_positions",
                 "nbody_destroy"):
        assert name in d


def test_library_exports_every_declared_symbol(lib):
    from paper_conf_sc_casselldahg24_b200 import _capi
    from paper_conf_sc_casselldahg24_b200.build import LIB
    out = subprocess.run(["nm", "-D", "--defined-only", LIB], capture_output=True, text=True, check=True).stdout
    exported = set(re.findall(r"\bT (nbody_[a-z_0-9]+)$", out, flags=re.M))
    for name in _declared():
        assert name in exported, name
        assert hasattr(lib, name)
    assert set(_capi.SIGNATURES) == set(_declared())


def test_library_is_sm100a(lib):
    from paper_conf_sc_casselldahg24_b200.build import LIB
    out = subprocess.run(["cuobjdump", "--list-elf", LIB], capture_output=True, text=True, check=True).stdout
    assert "sm_100a" in out


def test_host_side_argument_validation(lib):
    h = C.c_void_p()
    assert lib.nbody_create(0, 0.5, 1e-3, 1e-3, C.byref(h)) == -1 and not h.value
    assert lib.nbody_create(10, -0.1, 1e-3, 1e-3, C.byref(h)) == -1
    assert lib.nbody_create(10, float("nan"), 1e-3, 1e-3, C.byref(h)) == -1
    assert lib.nbody_create(10, 0.5, -1.0, 1e-3, C.byref(h)) == -1
    assert lib.nbody_create(1 << 30, 0.5, 1e-3, 1e-3, C.byref(h)) == -1
    assert lib.nbody_create(10, 0.5, 1e-3, 1e-3, None) == -1
    assert lib.nbody_set_option(None, 1, 16) == -1
    assert lib.nbody_step(None, 1) == -1
    assert lib.nbody_last_error(None) == b"null context"
    lib.nbody_destroy(None)
    assert lib.nbody_version() == 100


def test_oracle_and_cuda_path_share_nothing():
    """The oracle is test infrastructure: the CUDA sources never include or
    load it, and it never includes the CUDA sources."""
    for f in os.listdir(CSRC):
        txt = open(os.path.join(CSRC, f)).read()
        assert not re.search(r"#include[^\n]*oracle", txt), f
        assert "bvh_oracle" not in txt and "orc_" not in txt, f
    pkg = os.path.join(ROOT, "paper_conf_sc_casselldahg24_b200")
    for f in os.listdir(pkg):
        if f.endswith(".py"):
            assert "import oracle" not in open(os.path.join(pkg, f)).read()
            assert "from oracle" not in open(os.path.join(pkg, f)).read()
    otxt = open(os.path.join(ROOT, "oracle", "bvh_oracle.cpp")).read()
    assert "#include \"" not in otxt and "csrc" not in otxt.replace("paper_conf_sc_casselldahg24_b200/csrc", "")


def test_workspace_bytes_host_side(lib):
    """nbody_workspace_bytes is host-only (no device needed): one layout per N
    (sizes fixed by N), every world and key width; 0 on bad
    arguments; the optional buffers add their documented sizes."""
    from paper_conf_sc_casselldahg24_b200 import _capi
    f = lib.nbody_workspace_bytes
    fx = lib.nbody_workspace_bytes_ex
    for n in (1, 1000, 10_000_000):
        base = f(n, 1, 16)
        assert base > 0 and base % 256 == 0
        assert f(n, 8, 0) == base and f(n, 256, 21) == base
        L = max(0, (n - 1).bit_length())
        inner = 1 << L
        assert fx(n, 1, 16, _capi.NBODY_WS_QUAD) - base >= 80 * inner
        assert fx(n, 1, 16, _capi.NBODY_WS_XFER) - base >= 80 * n
        assert fx(n, 1, 16, _capi.NBODY_WS_FP64) - base >= 128 * n
        assert fx(n, 1, 16, 7) == (fx(n, 1, 16, 1) + fx(n, 1, 16, 2) + fx(n, 1, 16, 4) - 2 * base)
    # about 300 B of state + keys + sort per body and about 100 B per tree id at 10^7
    assert 3e9 < f(10_000_000, 1, 16) < 6e9
    assert f(2000, 1, 16) > f(1000, 1, 16)
    for bad in ((0, 1, 16), (1 << 30, 1, 16), (10, 0, 16), (10, 257, 16), (10, 1, 22), (10, 1, -1)):
        assert f(*bad) == 0
    assert fx(10, 1, 16, 8) == 0
    h = C.c_void_p()
    assert lib.nbody_create_ws(10, 0.5, 1e-3, 1e-3, None, 1 << 20, C.byref(h)) == -1 and not h.value
    assert lib.nbody_attach_comm(None, None, 0, 1) == -1


def test_concurrent_builds_do_not_race(tmp_path):
    """torchrun ranks (or test workers) that find the library stale at the
    same time: one process compiles under the build lock, the other waits and
    loads the result; neither fails on the other's temporary file."""
    import sys
    import textwrap
    lib = str(tmp_path / "libnbody_race.so")
    code = textwrap.dedent(f"""
        import sys
        sys.path.insert(0, {ROOT!r})
        from paper_conf_sc_casselldahg24_b200 import build as B
        B.LIB = {lib!r}
        B.build()
        import ctypes
        ctypes.CDLL(B.LIB).nbody_version
    """)
    procs = [subprocess.Popen([sys.executable, "-c", code]) for _ in range(2)]
    assert [p.wait(timeout=900) for p in procs] == [0, 0]
    assert os.path.exists(lib) and not [f for f in os.listdir(tmp_path) if f.endswith(".tmp")]
