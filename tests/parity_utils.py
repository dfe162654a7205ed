"""Helpers shared by the parity tests (comparison metrics only -- no method
arithmetic lives here)."""
import numpy as np

# BASELINE.json north star: accelerations within 1e-4 RMS relative error and
# every body within 1e-2 (same theta, eps, inputs).
ACC_RMS_TOL = 1e-4
ACC_MAX_TOL = 1e-2


def rel_errors(a_gpu, a_ref):
    """Per-body ||a_gpu - a_ref|| / ||a_ref|| (fp64), guarding exact zeros."""
    a_gpu = np.asarray(a_gpu, np.float64)
    a_ref = np.asarray(a_ref, np.float64)
    num = np.linalg.norm(a_gpu - a_ref, axis=1)
    den = np.linalg.norm(a_ref, axis=1)
    floor = 1e-30 + 1e-12 * float(np.sqrt(np.mean(den ** 2))) if len(den) else 1e-30
    return num / np.maximum(den, floor)


def assert_acc_close(a_gpu, a_ref, rms_tol=ACC_RMS_TOL, max_tol=ACC_MAX_TOL):
    e = rel_errors(a_gpu, a_ref)
    rms = float(np.sqrt(np.mean(e ** 2))) if len(e) else 0.0
    mx = float(e.max()) if len(e) else 0.0
    assert rms <= rms_tol and mx <= max_tol, f"acc rel error rms={rms:.3e} max={mx:.3e} (tol {rms_tol}, {max_tol})"
    return rms, mx
