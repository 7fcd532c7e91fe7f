"""Shared helpers of the GPU parity tests (no test functions here)."""
def rel_err_stats(y, want, bias=0.0):
    """max / median relative error of y against want, and of the bias-free
    parts (y - c_o against want - c_o): R17's output bias dilutes the relative
    error of the computed part."""
    import numpy as np
    y = np.asarray(y, np.float64)
    want = np.asarray(want, np.float64)
    r = np.abs(y - want) / np.abs(want)
    rb = np.abs(y - want) / np.abs(want - bias)
    return {"max_rel": float(r.max()), "median_rel": float(np.median(r)),
            "max_rel_nobias": float(rb.max()), "median_rel_nobias": float(np.median(rb)), "graphs": int(len(y))}
