"""Test infrastructure: an independent reference for the R30 horizon tables (R30), by direct
iteration of out^k over a bisection of float bit patterns -- no code shared with the library."""
import numpy as np


def range_thresholds(w0: float, b0: float, ymax: float, kmax: int = 32):
    """R30: out(m) = sigma(32-tap chain of the constant m, + b0), the map of a constant row
    through one uniform circulant layer.  thr_hi[k-1] = least m in [0, ymax] with out^k(m) == ymax,
    thr_lo[k-1] = greatest m with out^k(m) == 0, found here by direct iteration of out^k over a bisection
    of the float bit patterns (w0 is a power of two, so m*w0 is exact and the fp32 add is the fma)."""
    f32 = np.float32

    def out(m):
        acc = f32(0.0)
        for _ in range(32):
            acc = f32(acc + f32(m) * f32(w0))
        return float(min(max(f32(acc + f32(b0)), f32(0.0)), f32(ymax)))

    def outk(m, k):
        for _ in range(k):
            m = out(m)
        return m

    top = int(np.array(ymax, np.float32).view(np.uint32))
    flt = lambda u: float(np.array(u, np.uint32).view(np.float32))
    hi, lo = [], []
    for k in range(1, kmax + 1):
        a0, a1 = 0, top
        if outk(ymax, k) != ymax:
            hi.append(np.inf)
        else:
            while a0 < a1:
                mid = (a0 + a1) // 2
                a0, a1 = (a0, mid) if outk(flt(mid), k) == ymax else (mid + 1, a1)
            hi.append(flt(a0))
        a0, a1 = 0, top
        if outk(0.0, k) != 0.0:
            lo.append(-1.0)
        else:
            while a0 < a1:
                mid = (a0 + a1 + 1) // 2
                a0, a1 = (mid, a1) if outk(flt(mid), k) == 0.0 else (a0, mid - 1)
            lo.append(flt(a0))
    return hi, lo
