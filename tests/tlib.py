"""Shared test helpers (paths, GPU detection).  Imported as ``tlib`` (tests/ is on sys.path)."""
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden")


def has_gpu() -> bool:
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


def margin_bound(f) -> float:
    """Bound on |GPU fp64 value - oracle fp64 value| of a class decision (reading R3).

    Both sides add the same T leaf values (each an exact fp64 conversion of an fp32) in some
    order; any summation order of T terms errs by at most gamma_{T-1} * sum|v_t| with
    gamma_k = k u / (1 - k u), u = 2^-53 (Higham, Accuracy and Stability of Numerical Algorithms,
    §4.2), and sum|v_t| <= T * max|leaf value|.  The two sides' errors add, and a CLASS_SUM argmax
    compares two class sums, so the decision bound is 4 * gamma_T * T * max|v|."""
    import numpy as np
    leaves = f["feature"] < 0
    vmax = float(np.abs(f["leaf_value"][leaves]).max()) if leaves.any() else 0.0
    T = len(f["root"])
    u = 2.0 ** -53
    gamma = T * u / (1.0 - T * u)
    return 4.0 * gamma * T * vmax
