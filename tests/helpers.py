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
    # a NaN / inf output (e.g. a never-written element of a NaN-prefilled buffer) fails
    # here: otherwise |gpu - ref| / T is NaN and every comparison with it is False
    bad = ~np.isfinite(gpu) & np.isfinite(ref)
    if bad.any():
        idx = tuple(np.argwhere(bad)[0])
        raise AssertionError(f"{what}: non-finite output at {idx}: gpu={gpu[idx]!r} "
                             f"ref={ref[idx]!r} ({int(bad.sum())} such elements)")
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


# ------------------------------------------- occupancy, derived independently ----
# DTP's ActiveblocksPerSM (Eq. 3) is what the library asks the CUDA occupancy API
# for its SpMM kernel.  The tests re-derive it from the kernel's resource usage as
# cuobjdump reports it and the B200 per-SM limits, so a wrong occupancy query (or a
# wrong kernel picked for it) cannot pass by feeding the library's own value to the
# oracle.
B200_SM = dict(regs=65536, reg_unit=256, threads=2048, blocks=32, smem=233472)
_RES = None


def kernel_resources(lib_path):
    """{(kernel, TF, VW, L, R/V, VWS[, AGG]): (REG, SHARED)} from cuobjdump."""
    import re
    import subprocess
    global _RES
    if _RES is None:
        out = subprocess.run(["cuobjdump", "--dump-resource-usage", lib_path],
                             capture_output=True, text=True, check=True).stdout
        res, name = {}, None
        for line in out.splitlines():
            m = re.search(r"Function (\S+):", line)
            if m:
                name = m.group(1)
                continue
            m = re.search(r"REG:(\d+) .*SHARED:(\d+)", line)
            if m and name:
                k = re.search(r"(spmm|sddmm)_kernelINS_\d+(F32|BF16)E((?:Li\d+E)+)", name)
                if k:
                    ints = tuple(int(x) for x in re.findall(r"Li(\d+)E", k.group(3)))
                    res[(k.group(1), k.group(2)) + ints] = (int(m.group(1)), int(m.group(2)))
                name = None
        _RES = res
    return _RES


def expected_active_blocks(lib_path, dtype, vw, lanes, vecs, wpb):
    """Resident blocks/SM of spmm_kernel<dtype, vw, lanes, vecs, 1, sum> at wpb warps per
    block with the plan's tile smem (sized for 4-wide sparse vectors: 2 stages x 3 arrays
    x (32 / lanes) groups x (4 * lanes + 4) words per warp).  Rows of two
    vectors per lane on <= 16 lanes are launched as one vector per lane on twice the
    lanes ("widen"), so that is the kernel whose occupancy counts."""
    if vecs == 2 and lanes <= 16:
        lanes, vecs = 2 * lanes, 1
    regs, static_smem = kernel_resources(lib_path)[("spmm", dtype, vw, lanes, vecs, 1, 0)]
    S = B200_SM
    # the register file is split over the SM's 4 sub-partitions; a warp's registers
    # (allocated in 256-register units) come from one of them
    per_warp_regs = -(-regs * 32 // S["reg_unit"]) * S["reg_unit"]
    by_regs = (4 * ((S["regs"] // 4) // per_warp_regs)) // wpb
    dyn = wpb * 2 * 3 * (32 // lanes) * (4 * lanes + 4) * 4
    by_smem = S["smem"] // (dyn + static_smem)
    by_threads = S["threads"] // (32 * wpb)
    return min(by_regs, by_smem, by_threads, S["blocks"])


def independent_device_params(info, no_locality=False, **overrides):
    """(num_sms, active_blocks_per_sm, l2_bytes) for the oracle's plan, NOT taken from the
    library's plan info: torch's device properties and the cuobjdump-derived occupancy
    (or the test's explicit overrides, which the library was given too)."""
    import torch
    import paper_conf_ipps_fanwc23_b200 as gs
    prop = torch.cuda.get_device_properties(torch.cuda.current_device())
    nsm = overrides.get("num_sms") or prop.multi_processor_count
    dt = "BF16" if info["feature_dtype"] == 1 else "F32"
    abs_ = overrides.get("active_blocks_per_sm") or expected_active_blocks(
        gs.LIB_PATH, dt, info["vw_feat"], info["lanes"], info["vecs"], info["warps_per_block"])
    l2 = 0 if no_locality else (overrides.get("l2_bytes") or prop.L2_cache_size)
    return nsm, abs_, l2


def oracle_plan_checked(p, g, K, **kw):
    """The oracle's plan for the same inputs as library plan p (device parameters derived
    independently); asserts info and the three plan arrays are bit-exact."""
    import oracle
    info = p.info()
    nsm, abs_, l2 = independent_device_params(
        info, kw.get("no_locality", False), **{k: kw[k] for k in
                                               ("num_sms", "active_blocks_per_sm", "l2_bytes")
                                               if kw.get(k)})
    assert (info["num_sms"], info["active_blocks_per_sm"], info["l2_bytes"]) == (nsm, abs_, l2)
    dt = kw.get("feature_dtype", 0)
    ref = oracle.plan(g.row_ind, K, nsm, abs_, alpha=kw.get("alpha", 2) or 2,
                      warps_per_block=kw.get("warps_per_block") or 2,  # library default
                      force_chunk=kw.get("force_chunk", 0), force_vw=kw.get("force_vw", 0),
                      feature_dtype=1 if dt in (1, "bf16") else 0, M=g.M, l2_bytes=l2)
    assert info == ref.info, (info, ref.info)
    rf, rl, fl = (t.cpu().numpy() for t in p.arrays())
    assert np.array_equal(rf, ref.row_first)
    assert np.array_equal(rl, ref.row_last)
    assert np.array_equal(fl, ref.flags)
    return info
