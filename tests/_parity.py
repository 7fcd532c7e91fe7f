"""Shared helpers of the GPU parity tests (no test functions here)."""


def rel_err_stats(y, want, cond):
    """max / median relative error of y against want (north star: <= 2e-3),
    and of the bias-free part y - c_o (R17's output bias would dilute the
    first): |y - want| over cond = sum_i |w_o,i h2_i|, the magnitude of the
    terms of the head's last dot product (oracle.head_condition, reading R22)."""
    import numpy as np
    y = np.asarray(y, np.float64)
    want = np.asarray(want, np.float64)
    cond = np.asarray(cond, np.float64)
    r = np.abs(y - want) / np.abs(want)
    rb = np.abs(y - want) / cond
    return {"max_rel": float(r.max()), "median_rel": float(np.median(r)),
            "max_rel_nobias": float(rb.max()), "median_rel_nobias": float(np.median(rb)), "graphs": int(len(y))}
