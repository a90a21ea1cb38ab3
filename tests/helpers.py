"""Shared test helpers: tolerance checks and graph upload (no method arithmetic)."""
import numpy as np

TOL_FP32 = 1e-5  # BASELINE.json north_star: max|err| <= 1e-5 * sum|terms| per element


def assert_within(gpu, ref, T, tol=TOL_FP32, what=""):
    """|gpu - ref| <= tol * T elementwise; where T == 0 the GPU value must be +-0.
    Reports the worst err/T and its location on failure."""
    gpu = np.asarray(gpu, np.float64)
    ref = np.asarray(ref, np.float64)
    T = np.asarray(T, np.float64)
    assert gpu.shape == ref.shape == T.shape, (gpu.shape, ref.shape, T.shape)
    zero = T == 0
    if zero.any():
        assert (gpu[zero] == 0).all(), f"{what}: nonzero output where sum|terms| = 0"
    nz = ~zero
    if nz.any():
        ratio = np.abs(gpu[nz] - ref[nz]) / T[nz]
        worst = float(ratio.max())
        if worst > tol:
            idx = np.argwhere(nz)[int(ratio.argmax())]
            raise AssertionError(f"{what}: max err/T = {worst:.3e} > {tol:.0e} at {tuple(idx)}: "
                                 f"gpu={gpu[tuple(idx)]!r} ref={ref[tuple(idx)]!r}")
        return worst
    return 0.0


def upload(g, device="cuda", with_val=True, with_row_ptr=True):
    import paper_conf_ipps_fanwc23_b200 as gs
    return gs.DeviceGraph.from_arrays(g.M, g.N, g.row_ind, g.col_ind,
                                      g.val if with_val else None,
                                      g.row_ptr if with_row_ptr else None, device=device)
