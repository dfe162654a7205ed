"""Thin Python wrapper over the C ABI (include/nbody.h).

Arrays may be numpy arrays (host) or torch tensors (host or CUDA); they are
passed to the library by pointer.  PyTorch supplies device memory, streams
and process groups only -- every stage of the step runs in libnbody_b200.so.
"""
from __future__ import annotations

import ctypes as C

import numpy as np

from . import _capi


def _ptr(a) -> int:
    """Raw pointer of a C-contiguous numpy array or torch tensor."""
    if isinstance(a, np.ndarray):
        if not a.flags["C_CONTIGUOUS"]:
            raise ValueError("array must be C-contiguous")
        return a.ctypes.data
    if hasattr(a, "data_ptr"):
        if not a.is_contiguous():
            raise ValueError("tensor must be contiguous")
        return a.data_ptr()
    if isinstance(a, int):
        return a
    raise TypeError(f"unsupported buffer type {type(a)}")


def _f64(a, n, cols):
    if isinstance(a, np.ndarray):
        a = np.ascontiguousarray(a, dtype=np.float64)
        if a.size != n * cols:
            raise ValueError(f"expected {n}x{cols} values, got {a.shape}")
        return a
    if hasattr(a, "data_ptr"):
        import torch
        if a.dtype != torch.float64 or a.numel() != n * cols:
            raise ValueError("expected a float64 tensor of n*cols elements")
        return a.contiguous()
    raise TypeError(type(a))


def _f32(a, n, cols):
    if isinstance(a, np.ndarray):
        a = np.ascontiguousarray(a, dtype=np.float32)
        if a.size != n * cols:
            raise ValueError(f"expected {n}x{cols} values, got {a.shape}")
        return a
    if hasattr(a, "data_ptr"):
        import torch
        if a.dtype != torch.float32 or a.numel() != n * cols:
            raise ValueError("expected a float32 tensor of n*cols elements")
        return a.contiguous()
    raise TypeError(type(a))


class NBody:
    """One simulation context: ``NBody(n, theta, eps, dt)``."""

    def __init__(self, n: int, theta: float = 0.5, eps: float = 1e-3, dt: float = 1e-3, *, key_bits: int = 16,
                 stream=None, use_graph: bool = True, traversal: int = 0, device=None, multipole: int = 1,
                 balance: bool = False, precision: int = 32, workspace=None):
        """``workspace``: optional caller-owned device buffer (a CUDA uint8
        torch tensor, at least ``NBody.workspace_bytes(n, ...)`` bytes) the
        context carves all its device memory from (nbody_create_ws); the
        caller keeps it alive while the context lives."""
        self.lib = _capi.load()
        self.n = int(n)
        if device is None:  # follow PyTorch's current device when torch has one
            try:
                import torch
                if torch.cuda.is_available():
                    device = torch.cuda.current_device()
            except ImportError:
                pass
        if device is not None:
            st = self.lib.nbody_select_device(int(device))
            if st != 0:
                raise _capi.NBodyError(st, f"nbody_select_device({device}) failed")
        h = C.c_void_p()
        if workspace is None:
            st = self.lib.nbody_create(self.n, float(theta), float(eps), float(dt), C.byref(h))
        else:
            nbytes = workspace.numel() * workspace.element_size()
            st = self.lib.nbody_create_ws(self.n, float(theta), float(eps), float(dt), _ptr(workspace), nbytes,
                                          C.byref(h))
        if st != 0:
            raise _capi.NBodyError(st, "nbody_create failed" if workspace is None else "nbody_create_ws failed")
        self.workspace = workspace
        self.h = h
        self.set_option(_capi.NBODY_OPT_KEY_BITS, key_bits)
        self.set_option(_capi.NBODY_OPT_USE_GRAPH, int(use_graph))
        self.set_option(_capi.NBODY_OPT_TRAVERSAL, traversal)
        if multipole != 1:
            self.set_option(_capi.NBODY_OPT_MULTIPOLE, multipole)
        if balance:  # NEXT-3(i) cost-weighted ranges (peer exchange only)
            self.set_option(_capi.NBODY_OPT_BALANCE, 1)
        self.precision = int(precision)
        if self.precision != 32:  # NEXT-2 FP64 mode
            self.set_option(_capi.NBODY_OPT_PRECISION, self.precision)
        if stream is not None:
            self.set_option(_capi.NBODY_OPT_STREAM, int(stream))

    @staticmethod
    def workspace_bytes(n: int, world: int = 1, key_bits: int = 16, features: int = 0) -> int:
        """Device bytes a context for n bodies needs (nbody_workspace_bytes_ex);
        features: NBODY_WS_QUAD | NBODY_WS_XFER | NBODY_WS_FP64."""
        b = _capi.load().nbody_workspace_bytes_ex(int(n), int(world), int(key_bits), int(features))
        if b == 0:
            raise ValueError("invalid arguments to nbody_workspace_bytes_ex")
        return int(b)

    # -- lifecycle ---------------------------------------------------------
    def close(self):
        if getattr(self, "h", None):
            self.lib.nbody_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def _ck(self, st):
        _capi.check(self.h, st)

    # -- calls -------------------------------------------------------------
    def set_option(self, opt: int, value: int):
        self._ck(self.lib.nbody_set_option(self.h, int(opt), int(value)))

    def set_bodies(self, pos, vel, mass):
        if self.precision == 64:
            p, v, m = _f64(pos, self.n, 3), _f64(vel, self.n, 3), _f64(mass, self.n, 1)
            self._ck(self.lib.nbody_set_bodies64(self.h, _ptr(p), _ptr(v), _ptr(m)))
            return
        p, v, m = _f32(pos, self.n, 3), _f32(vel, self.n, 3), _f32(mass, self.n, 1)
        self._ck(self.lib.nbody_set_bodies(self.h, _ptr(p), _ptr(v), _ptr(m)))

    def set_bodies_async(self, pos, vel, mass):
        """nbody_set_bodies_async: the copy runs on the copy stream and overlaps
        queued steps; `pos`, `vel`, `mass` (pinned host or device, fp32,
        contiguous) must stay unchanged until sync()."""
        if self.precision == 64:
            raise ValueError("set_bodies_async is fp32 only")
        self._keep_in = (_f32(pos, self.n, 3), _f32(vel, self.n, 3), _f32(mass, self.n, 1))
        p, v, m = self._keep_in
        self._ck(self.lib.nbody_set_bodies_async(self.h, _ptr(p), _ptr(v), _ptr(m)))

    def get_positions_async(self, out):
        """nbody_get_positions_async into out[n][3] (pinned host or device fp32,
        contiguous); valid after sync()."""
        o = _f32(out, self.n, 3)
        if _ptr(o) != _ptr(out):
            raise ValueError("get_positions_async needs a contiguous float32 [n, 3] output")
        self._ck(self.lib.nbody_get_positions_async(self.h, _ptr(o)))

    def compute_accel(self):
        self._ck(self.lib.nbody_compute_accel(self.h))

    def step(self, nsteps: int = 1):
        self._ck(self.lib.nbody_step(self.h, int(nsteps)))

    def sync(self):
        self._ck(self.lib.nbody_sync(self.h))

    def _get3(self, fn, out=None):
        out = np.empty((self.n, 3), np.float32) if out is None else out
        self._ck(fn(self.h, _ptr(out)))
        return out

    def get_accel(self, out=None):
        return self._get3(self.lib.nbody_get_accel, out)

    def get_positions(self, out=None):
        return self._get3(self.lib.nbody_get_positions, out)

    def get_velocities(self, out=None):
        return self._get3(self.lib.nbody_get_velocities, out)

    # NEXT-2 FP64 mode getters
    def _get3d(self, fn, out=None):
        out = np.empty((self.n, 3), np.float64) if out is None else out
        self._ck(fn(self.h, _ptr(out)))
        return out

    def get_accel64(self, out=None):
        return self._get3d(self.lib.nbody_get_accel64, out)

    def get_positions64(self, out=None):
        return self._get3d(self.lib.nbody_get_positions64, out)

    def get_velocities64(self, out=None):
        return self._get3d(self.lib.nbody_get_velocities64, out)

    def get_state64(self):
        pm = np.empty((self.n, 4), np.float64)
        vi = np.empty((self.n, 4), np.float64)
        self._ck(self.lib.nbody_get_state64(self.h, _ptr(pm), _ptr(vi)))
        return pm, vi

    def debug_level64(self, level: int):
        cnt = C.c_int64()
        self._ck(self.lib.nbody_debug_level64(self.h, int(level), C.byref(cnt), None, None))
        rec = np.empty((cnt.value, 4), np.float64)
        box = np.empty((cnt.value, 6), np.float64)
        self._ck(self.lib.nbody_debug_level64(self.h, int(level), C.byref(cnt), _ptr(rec), _ptr(box)))
        return rec, box

    def get_interactions(self, out=None):
        out = np.empty(self.n, np.uint32) if out is None else out
        self._ck(self.lib.nbody_get_interactions(self.h, _ptr(out)))
        return out

    def get_state(self):
        pm = np.empty((self.n, 4), np.float32)
        vi = np.empty((self.n, 4), np.float32)
        self._ck(self.lib.nbody_get_state(self.h, _ptr(pm), _ptr(vi)))
        return pm, vi

    def set_state(self, pos_m, vel_id, steps: int = 0):
        """Checkpoint restore (nbody_set_state / nbody_set_state64): the slot-order
        state of get_state() / get_state64() with its ids, and the step counter
        (stats()["steps"] of the checkpointed context)."""
        if self.precision == 64:
            p, v = _f64(pos_m, self.n, 4), _f64(vel_id, self.n, 4)
            self._ck(self.lib.nbody_set_state64(self.h, _ptr(p), _ptr(v), int(steps)))
            return
        p, v = _f32(pos_m, self.n, 4), _f32(vel_id, self.n, 4)
        self._ck(self.lib.nbody_set_state(self.h, _ptr(p), _ptr(v), int(steps)))

    def stats(self) -> dict:
        s = _capi.nbody_stats()
        self._ck(self.lib.nbody_get_stats(self.h, C.byref(s)))
        return {f: getattr(s, f) for f, _ in s._fields_}

    def direct_accel(self, ids):
        """Exact fp64 direct-sum accelerations (NEXT-1) for the given body ids."""
        ids = np.ascontiguousarray(ids, np.int64)
        out = np.empty((len(ids), 3), np.float64)
        self._ck(self.lib.nbody_direct_accel(self.h, _ptr(ids), len(ids), _ptr(out)))
        return out

    def allpairs_accel(self, ids, timed: bool = False):
        """NEXT-1 fp32 all-pairs accelerations (fp64 output) of the given body
        ids against all n sources; with timed=True also the kernel's device
        time in ms."""
        if hasattr(ids, "data_ptr"):  # a torch tensor (host or device): int64, contiguous
            import torch
            if ids.dtype != torch.int64:
                raise ValueError("ids must be int64")
            ids = ids.contiguous()
        else:
            ids = np.ascontiguousarray(ids, np.int64)
        out = np.empty((len(ids), 3), np.float64)
        ms = C.c_float(0.0)
        self._ck(self.lib.nbody_allpairs_accel(self.h, _ptr(ids), len(ids), _ptr(out),
                                               C.byref(ms) if timed else None))
        return (out, ms.value) if timed else out

    # -- multi-GPU ---------------------------------------------------------
    def set_partition(self, rank: int, world: int):
        self._ck(self.lib.nbody_set_partition(self.h, int(rank), int(world)))

    def partition(self):
        r, w = C.c_int(), C.c_int()
        b, e = C.c_int64(), C.c_int64()
        self._ck(self.lib.nbody_get_partition(self.h, C.byref(r), C.byref(w), C.byref(b), C.byref(e)))
        return r.value, w.value, b.value, e.value

    def copy_owned_from(self, other: "NBody"):
        self._ck(self.lib.nbody_copy_owned(self.h, other.h))

    def attach_nccl(self, unique_id: bytes, rank: int, world: int):
        buf = C.create_string_buffer(bytes(unique_id), 128)
        self._ck(self.lib.nbody_attach_nccl(self.h, buf, int(rank), int(world)))

    def attach_process_group(self, rank: int, world: int, group=None):
        """Bootstrap the library's NCCL communicator through torch.distributed:
        rank 0 creates the unique id, the process group broadcasts it."""
        from .dist import broadcast_unique_id
        self.attach_nccl(broadcast_unique_id(rank, group), rank, world)

    def attach_comm(self, comm_ptr: int, rank: int, world: int):
        """Run the exchange on an existing ncclComm_t (nbody_attach_comm)."""
        self._ck(self.lib.nbody_attach_comm(self.h, C.c_void_p(int(comm_ptr)), int(rank), int(world)))

    def attach_torch_comm(self, group=None):
        """Use torch.distributed's own NCCL communicator of this device (the
        process group must be NCCL and eagerly initialised with device_id)."""
        import torch
        import torch.distributed as dist
        g = group if group is not None else dist.group.WORLD
        backend = g._get_backend(torch.device("cuda", torch.cuda.current_device()))
        self.attach_comm(backend._comm_ptr(), dist.get_rank(g), dist.get_world_size(g))

    # fused update + exchange over peer memory (nbody_attach_peers)
    def peer_handle(self) -> bytes:
        buf = C.create_string_buffer(128)
        self._ck(self.lib.nbody_peer_handle(self.h, buf))
        return buf.raw

    def attach_peers(self, handles, rank: int, world: int):
        """handles: the world 128-byte descriptors indexed by rank."""
        blob = b"".join(bytes(h) for h in handles)
        if len(blob) != 128 * world:
            raise ValueError("need world descriptors of 128 bytes")
        buf = C.create_string_buffer(blob, len(blob))
        self._ck(self.lib.nbody_attach_peers(self.h, buf, int(rank), int(world)))

    def attach_peers_group(self, rank: int, world: int, group=None):
        """Gather the descriptors over a torch.distributed group and attach."""
        import torch.distributed as dist
        handles = [None] * world
        dist.all_gather_object(handles, self.peer_handle(), group=group)
        self.attach_peers(handles, rank, world)

    @staticmethod
    def attach_peers_local(bodies):
        """Contexts of one process (bodies[r] becomes rank r)."""
        lib = _capi.load()
        arr = (C.c_void_p * len(bodies))(*[b.h.value for b in bodies])
        st = lib.nbody_attach_peers_local(arr, len(bodies))
        if st != 0:
            raise _capi.NBodyError(st, "nbody_attach_peers_local: " + "; ".join(
                lib.nbody_last_error(b.h).decode() for b in bodies if lib.nbody_last_error(b.h)))

    def exchange_mode(self) -> str:
        return {0: "none", 1: "nccl", 2: "peer"}[self.lib.nbody_exchange_mode(self.h)]

    # -- debug views (parity tests) -----------------------------------------
    def debug_keys(self):
        out = np.empty(self.n, np.uint64)
        self._ck(self.lib.nbody_debug_keys(self.h, _ptr(out)))
        return out

    def debug_perm(self):
        out = np.empty(self.n, np.uint32)
        self._ck(self.lib.nbody_debug_perm(self.h, _ptr(out)))
        return out

    def debug_quad(self, level: int):
        cnt = C.c_int64()
        self._ck(self.lib.nbody_debug_level(self.h, int(level), C.byref(cnt), None, None, None))
        out = np.empty((cnt.value, 6), np.float64)
        self._ck(self.lib.nbody_debug_quad(self.h, int(level), _ptr(out)))
        return out

    def debug_level(self, level: int):
        cnt = C.c_int64()
        self._ck(self.lib.nbody_debug_level(self.h, int(level), C.byref(cnt), None, None, None))
        c = cnt.value
        pred = np.empty((c, 4), np.float64)
        rec = np.empty((c, 4), np.float32)
        box = np.empty((c, 6), np.float32) if self.precision == 32 else None  # fp64: debug_level64
        self._ck(self.lib.nbody_debug_level(self.h, int(level), C.byref(cnt), _ptr(pred), _ptr(rec),
                                            _ptr(box) if box is not None else None))
        return pred, rec, box
