"""Pins for oracle/be.py (c3-c10): closed forms, invariants, special cases and brute force on
tiny inputs, chosen so a dropped term / wrong sign / wrong index fails one of them."""
import cmath
import math

import numpy as np
import pytest

import synth
from oracle import be
from oracle.metrics import max_rel_err

C0, C1 = np.float32(1.0 / 6.0), np.float32(1.0 / 36.0)


# ------------------------------------------------------------------ sgemm
def test_sgemm_bruteforce_and_identity():
    A, B = synth.sgemm_inputs(5, 7, 6, seed=1, variant="int")
    C, S = be.sgemm(A, B)
    ref = np.array([[sum(float(A[i, k]) * float(B[k, j]) for k in range(6)) for j in range(7)] for i in range(5)])
    assert np.array_equal(C, ref)
    I = np.eye(6, dtype=np.float32)
    C2, _ = be.sgemm(A[:, :6], I)
    assert np.array_equal(C2, A[:, :6].astype(np.float64))


def test_sgemm_alpha_beta():
    A, B = synth.sgemm_inputs(3, 4, 2, seed=2, variant="int")
    Cin = np.full((3, 4), 2.0, np.float32)
    C, _ = be.sgemm(A, B, alpha=2.0, beta=-0.5, C_in=Cin)
    assert np.array_equal(C, 2.0 * (A.astype(np.float64) @ B.astype(np.float64)) - 1.0)


def test_sgemm_orientation():
    A = np.array([[1, 2, 3]], np.float32)          # 1x3
    B = np.array([[1], [10], [100]], np.float32)   # 3x1
    C, _ = be.sgemm(A, B)
    assert C.shape == (1, 1) and C[0, 0] == 321.0


# ------------------------------------------------------------------ stencil
def test_stencil_impulse_response():
    A = np.zeros((5, 6, 7), np.float32)
    A[2, 3, 3] = 1.0
    An, _ = be.stencil(A, C0, C1)
    exp = np.zeros_like(An)
    exp[2, 3, 3] = -float(C0)
    for dz, dy, dx in [(1, 0, 0), (-1, 0, 0), (0, 1, 0), (0, -1, 0), (0, 0, 1), (0, 0, -1)]:
        exp[2 + dz, 3 + dy, 3 + dx] = float(C1)
    assert np.array_equal(An, exp)


def test_stencil_boundary_copied_and_linear_field_vanishes():
    z, y, x = np.meshgrid(np.arange(6), np.arange(7), np.arange(8), indexing="ij")
    A = (0.5 * x + 0.25 * y - 0.125 * z + 3.0).astype(np.float32)
    An, S = be.stencil(A, np.float64(1 / 6), np.float64(1 / 36))
    inner = An[1:-1, 1:-1, 1:-1]
    assert np.max(np.abs(inner) / S[1:-1, 1:-1, 1:-1]) < 1e-14     # 6*c1 == c0
    mask = np.ones(A.shape, bool)
    mask[1:-1, 1:-1, 1:-1] = False
    assert np.array_equal(An[mask], A[mask].astype(np.float64))


def test_stencil_bruteforce_dyadic():
    A = synth.stencil_inputs(6, 5, 4, seed=3, variant="dyadic")
    c0, c1 = 0.5, 1.0 / 16
    An, _ = be.stencil(A, c0, c1)
    nz, ny, nx = A.shape
    for zz in range(nz):
        for yy in range(ny):
            for xx in range(nx):
                if 0 < zz < nz - 1 and 0 < yy < ny - 1 and 0 < xx < nx - 1:
                    v = c1 * (float(A[zz, yy, xx - 1]) + float(A[zz, yy, xx + 1]) + float(A[zz, yy - 1, xx])
                              + float(A[zz, yy + 1, xx]) + float(A[zz - 1, yy, xx]) + float(A[zz + 1, yy, xx])) \
                        - c0 * float(A[zz, yy, xx])
                else:
                    v = float(A[zz, yy, xx])
                assert An[zz, yy, xx] == v


# ------------------------------------------------------------------ mri-q
def test_mriq_phimag():
    pm, _ = be.mriq_phimag(np.array([3.0, 0.5]), np.array([4.0, -0.5]))
    assert np.array_equal(pm, np.array([25.0, 0.5]))


def test_mriq_origin_and_zero_k():
    d = synth.mriq_inputs(8, 64, seed=4)
    pm, _ = be.mriq_phimag(d["phiR"], d["phiI"])
    # origin voxel (index of x=y=z=0) sees exp(0) for every k
    o = np.nonzero((d["x"] == 0) & (d["y"] == 0) & (d["z"] == 0))[0][0]
    Qr, Qi, _, _ = be.mriq_q(d["x"], d["y"], d["z"], d["kx"], d["ky"], d["kz"], pm)
    assert abs(Qr[o] - pm.sum()) < 1e-12 and abs(Qi[o]) < 1e-12
    z = np.zeros(64, np.float32)
    Qr0, Qi0, _, _ = be.mriq_q(d["x"], d["y"], d["z"], z, z, z, pm)
    assert np.allclose(Qr0, pm.sum(), rtol=0, atol=1e-12) and np.allclose(Qi0, 0, atol=1e-12)


def test_mriq_symmetric_k_has_zero_imag():
    d = synth.mriq_inputs(6, 32, seed=5)
    kx = np.concatenate([d["kx"], -d["kx"]])
    ky = np.concatenate([d["ky"], -d["ky"]])
    kz = np.concatenate([d["kz"], -d["kz"]])
    pm = np.concatenate([d["phiR"] ** 2, d["phiR"] ** 2])
    Qr, Qi, Sr, Si = be.mriq_q(d["x"], d["y"], d["z"], kx, ky, kz, pm)
    assert np.max(np.abs(Qi) / np.maximum(Si, 1e-30)) < 1e-12


def test_mriq_dirichlet_closed_form():
    # 1-D uniform k grid k_m = m*dk (m < M) along x, phiMag = 1: sum cos(2 pi m dk x)
    # = sin(pi M dk x) cos(pi (M-1) dk x) / sin(pi dk x)  (2*pi taken as the fp32 constant)
    M, dk = 40, 0.37
    x = np.array([0.013, 0.21, -0.4], np.float64)
    kx = np.arange(M) * dk
    zero = np.zeros(M)
    Qr, Qi, _, _ = be.mriq_q(x, np.zeros(3), np.zeros(3), kx, zero, zero, np.ones(M))
    th = be.TWO_PI_F32 / 2 * dk * x
    expr = np.sin(M * th) * np.cos((M - 1) * th) / np.sin(th)
    expi = np.sin(M * th) * np.sin((M - 1) * th) / np.sin(th)
    assert np.allclose(Qr, expr, rtol=1e-11, atol=1e-11)
    assert np.allclose(Qi, expi, rtol=1e-11, atol=1e-11)


def test_mriq_bruteforce_small_and_accumulate():
    d = synth.mriq_inputs(4, 16, seed=6)
    pm, _ = be.mriq_phimag(d["phiR"], d["phiI"])
    Qr, Qi, _, _ = be.mriq_q(d["x"], d["y"], d["z"], d["kx"], d["ky"], d["kz"], pm)
    for v in range(d["x"].size):
        r = i = 0.0
        for k in range(16):
            a = be.TWO_PI_F32 * (float(d["kx"][k]) * float(d["x"][v]) + float(d["ky"][k]) * float(d["y"][v])
                                 + float(d["kz"][k]) * float(d["z"][v]))
            r += float(pm[k]) * math.cos(a)
            i += float(pm[k]) * math.sin(a)
        assert abs(Qr[v] - r) < 1e-10 and abs(Qi[v] - i) < 1e-10
    # two chunks accumulate to the single pass
    a1 = be.mriq_q(d["x"], d["y"], d["z"], d["kx"][:7], d["ky"][:7], d["kz"][:7], pm[:7])
    a2 = be.mriq_q(d["x"], d["y"], d["z"], d["kx"][7:], d["ky"][7:], d["kz"][7:], pm[7:], a1[0], a1[1])
    assert np.allclose(a2[0], Qr, atol=1e-12) and np.allclose(a2[1], Qi, atol=1e-12)


# ------------------------------------------------------------------ cutcp
def test_cutcp_single_atom_closed_form():
    atoms = np.array([[2.3, 3.1, 1.7, 0.8]], np.float32)
    nx = ny = nz = 12
    h = 0.5
    V, _ = be.cutcp(atoms, nx, ny, nz, h, cutoff=4.0, excl=1.0)
    ax, ay, az, q = (float(v) for v in atoms[0])
    for f in range(nx * ny * nz):
        i, j, k = f % nx, (f // nx) % ny, f // (nx * ny)
        d = math.sqrt((i * h - ax) ** 2 + (j * h - ay) ** 2 + (k * h - az) ** 2)
        if d < 1.0 or d >= 4.0:
            exp = 0.0
        else:
            exp = q / d * (1 - d * d / 16.0) ** 2
        assert abs(V[f] - exp) < 1e-12


def test_cutcp_linear_in_charge_and_exclusion():
    d = synth.cutcp_inputs(6.0, seed=7)
    at = d["atoms"]
    V, _ = be.cutcp(at, d["nx"], d["ny"], d["nz"], 0.5, cutoff=4.0)
    a1 = at.copy(); a1[:, 3] *= 0.25
    a2 = at.copy(); a2[:, 3] *= 0.75
    V1, _ = be.cutcp(a1, d["nx"], d["ny"], d["nz"], 0.5, cutoff=4.0)
    V2, _ = be.cutcp(a2, d["nx"], d["ny"], d["nz"], 0.5, cutoff=4.0)
    assert np.allclose(V1 + V2, V, atol=1e-12)
    # exclusion: every point within 1 A of an atom is exactly 0
    pts = np.arange(d["nx"] ** 3)
    gi, gj, gk = pts % d["nx"], (pts // d["nx"]) % d["ny"], pts // (d["nx"] * d["ny"])
    g = np.stack([gi, gj, gk], 1) * 0.5
    dmin = np.min(np.linalg.norm(g[:, None, :] - at[None, :, :3].astype(np.float64), axis=2), axis=1)
    assert np.all(V[dmin < 1.0] == 0.0)
    assert np.all(np.abs(dmin - 1.0) > 1e-4)  # generator keeps exclusion decisions tie-free


def test_cutcp_points_subset():
    d = synth.cutcp_inputs(5.0, seed=8)
    V, _ = be.cutcp(d["atoms"], d["nx"], d["ny"], d["nz"], 0.5)
    pts = np.array([0, 17, 333, d["nx"] ** 3 - 1])
    Vs, _ = be.cutcp(d["atoms"], d["nx"], d["ny"], d["nz"], 0.5, points=pts)
    assert np.array_equal(Vs, V[pts])


# ------------------------------------------------------------------ lbm
def test_lbm_rest_equilibrium_is_fixed_point():
    f, fl = synth.lbm_inputs(6, 5, 7, seed=9, variant="rest")
    fl[:] = synth.LBM_FLUID
    dst, _ = be.lbm_step(f, fl, np.zeros_like(f))
    m = be.lbm_written_mask(6, 5, 7)
    # fixed point up to the fp32 rounding of the stored weights (|rho - 1| ~ 1e-8)
    assert np.max(np.abs(dst[m] - f.astype(np.float64)[m]) / f.astype(np.float64)[m]) < 1e-7


def test_lbm_collision_conserves_mass_and_momentum():
    f, fl = synth.lbm_inputs(8, 8, 8, seed=10)
    fl[:] = synth.LBM_FLUID
    dst, _ = be.lbm_step(f, fl, np.zeros_like(f))
    # pull back the post-collision values of one interior cell x from dst_i[x + e_i]
    x = (4, 4, 4)
    post = np.array([dst[i, x[0] + be.LBM_E[i, 2], x[1] + be.LBM_E[i, 1], x[2] + be.LBM_E[i, 0]] for i in range(19)])
    pre = f[:, x[0], x[1], x[2]].astype(np.float64)
    assert abs(post.sum() - pre.sum()) < 1e-13
    for a in range(3):
        assert abs((post * be.LBM_E[:, a]).sum() - (pre * be.LBM_E[:, a]).sum()) < 1e-13
    # and the equilibrium is reached with weight omega: post = pre + omega (feq - pre) != pre
    assert np.max(np.abs(post - pre)) > 0


def test_lbm_obstacle_bounce_back_is_copy_and_mass_is_conserved():
    nx, ny, nz = 7, 6, 8
    f, fl = synth.lbm_inputs(nx, ny, nz, seed=11)
    dst, _ = be.lbm_step(f, fl, np.zeros_like(f))
    # obstacle cell at a corner-free face position: its pushes are reflected copies
    z, y, x = 0, 3, 3
    for i in range(19):
        j = be.lbm_opposite(i)
        ex, ey, ez = be.LBM_E[j]
        tz, ty, tx = z + ez, y + ey, x + ex
        if 0 <= tz < nz and 0 <= ty < ny and 0 <= tx < nx:
            assert dst[j, tz, ty, tx] == float(f[i, z, y, x])
    # total mass: every value pushed to an in-grid destination; ACCEL cells change momentum but
    # collision still conserves mass, so sum(dst written) == sum(src) - discarded pushes
    m = be.lbm_written_mask(nx, ny, nz)
    fl64 = f.astype(np.float64)
    total_in = fl64.sum()
    total_out = dst[m].sum()
    # boundary cells are all obstacles; their outward reflected pushes leave the grid.
    disc = 0.0
    for i in range(19):
        j = be.lbm_opposite(i)
        ex, ey, ez = be.LBM_E[j]
        for zz in range(nz):
            for yy in range(ny):
                for xx in range(nx):
                    if fl[zz, yy, xx] == synth.LBM_OBSTACLE:
                        tz, ty, tx = zz + ez, yy + ey, xx + ex
                        if not (0 <= tz < nz and 0 <= ty < ny and 0 <= tx < nx):
                            disc += fl64[i, zz, yy, xx]
    assert abs(total_out - (total_in - disc)) < 1e-10 * total_in


def test_lbm_written_mask_counts():
    m = be.lbm_written_mask(4, 5, 6)
    assert m[0].all()
    assert m[3].sum() == 3 * 5 * 6   # E direction: x = 0 has no upstream
    assert m[7].sum() == 3 * 4 * 6   # NE


# ------------------------------------------------------------------ spmv
def test_jds_structure_and_spmv():
    row_ptr, cols, vals, x = synth.spmv_inputs(300, seed=12, mean_len=8)
    perm, rl, jptr, jcol, jval = be.jds_build(row_ptr, cols, vals)
    lens = np.diff(row_ptr)
    assert sorted(perm.tolist()) == list(range(300))
    for i in range(299):   # non-increasing length, ties by ascending row index (stable)
        assert rl[i] >= rl[i + 1]
        if rl[i] == rl[i + 1]:
            assert perm[i] < perm[i + 1]
    assert np.array_equal(rl, lens[perm])
    for d in range(len(jptr) - 1):
        assert jptr[d + 1] - jptr[d] == int((lens > d).sum())
    y, S = be.spmv_jds(perm, rl, jptr, jcol, jval, x)
    y2 = be.spmv_csr(row_ptr, cols, vals, x)
    assert max_rel_err(y2, y, S) < 1e-13
    # closed-form invariant: sum_r y_r = sum_c colsum_c x_c
    colsum = np.zeros(300)
    np.add.at(colsum, cols, vals.astype(np.float64))
    assert abs(y.sum() - (colsum * x).sum()) < 1e-9


def test_spmv_identity_and_permutation():
    for variant in ("identity", "perm"):
        row_ptr, cols, vals, x = synth.spmv_inputs(64, seed=13, variant=variant)
        jds = be.jds_build(row_ptr, cols, vals)
        y, _ = be.spmv_jds(*jds, x)
        assert np.array_equal(y, x.astype(np.float64)[cols])


# ------------------------------------------------------------------ histo
@pytest.mark.parametrize("variant", ["skewed", "uniform"])
def test_histo_sums_to_n(variant):
    v = synth.histo_inputs(100_000, 4096, seed=14, variant=variant)
    c = be.histo(v, 4096)
    assert int(c.astype(np.int64).sum()) == v.size


def test_histo_constant_and_each():
    v = synth.histo_inputs(5000, 4096, seed=15, variant="constant")
    c = be.histo(v, 4096)
    assert c[4096 // 3] == 5000 and c.sum() == 5000
    v = synth.histo_inputs(4096 * 7, 4096, seed=16, variant="each")
    assert np.all(be.histo(v, 4096) == 7)
    s = be.histo_saturate(np.array([0, 255, 256, 70000]))
    assert s.tolist() == [0, 255, 255, 255]


# ------------------------------------------------------------------ bfs
def test_bfs_path_star_two():
    rp, c = synth.bfs_inputs(10, 0, "path")
    assert be.bfs_levels(rp, c).tolist() == list(range(10))
    rp, c = synth.bfs_inputs(10, 0, "star")
    assert be.bfs_levels(rp, c).tolist() == [0] + [1] * 9
    rp, c = synth.bfs_inputs(10, 0, "two")
    assert be.bfs_levels(rp, c).tolist() == [0, 1, 2, 3, 4] + [-1] * 5


def test_bfs_two_kernel_levels_match_queue_bfs():
    rp, col = synth.bfs_inputs(2000, seed=17)
    V = 2000
    level = np.full(V, -1, np.int32); level[0] = 0
    mask = np.zeros(V, np.uint8); mask[0] = 1
    visited = mask.copy()
    upd = np.zeros(V, np.uint8)
    over = 1
    while over:
        level, mask, upd = be.bfs_expand(rp, col, level, mask, visited, upd)
        mask, visited, upd, over = be.bfs_commit(mask, visited, upd)
    assert np.array_equal(level, be.bfs_levels(rp, col))


# ------------------------------------------------------------------ fma_burn
def test_fma_burn_closed_form_matches_iteration():
    out = be.fma_burn(200, 37)
    for g in (0, 5, 96, 97, 199):
        s = 0.0
        for j in range(4):
            x = ((g % 97) + j) / 128.0
            for _ in range(37):
                x = x * 0.5 + 0.125 * (j + 1)
            s += x
        assert abs(out[g] - s) < 1e-14


def test_cutcp_bins_partition_atoms_in_index_order():
    d = synth.cutcp_inputs(9.0, seed=20)
    at = d["atoms"]
    bdim = ((d["nx"] + 7) // 8, (d["ny"] + 7) // 8, (d["nz"] + 7) // 8)
    bins, count = be.cutcp_bins(at, bdim, 4.0, 64)
    assert count.sum() == at.shape[0] and count.max() <= 64
    seen = []
    for b in range(bins.shape[0]):
        rows = bins[b, :count[b]]
        for r in rows:
            # every atom lies inside its bin's box
            ix, iy, iz = (int(np.floor(r[c] / 4.0)) for c in range(3))
            assert (iz * bdim[1] + iy) * bdim[0] + ix == b
        idx = [int(np.nonzero(np.all(at == r, axis=1))[0][0]) for r in rows]
        assert idx == sorted(idx)           # index order within a bin
        seen += idx
        assert np.all(bins[b, count[b]:, 3] == 0)
    assert sorted(seen) == list(range(at.shape[0]))


# ------------------------------------------------------------------ NEXT-3 mri-fhd (reading 14)
def test_mrifhd_rhophi_is_conj_phi_times_d():
    # RhoPhi = conj(phi) * d as a complex product (an independent formulation)
    g = np.random.default_rng(3)
    pr, pi, dr, di = (g.uniform(-1, 1, 50) for _ in range(4))
    rr, ri, sr, si = be.mrifhd_rhophi(pr, pi, dr, di)
    ref = np.conj(pr + 1j * pi) * (dr + 1j * di)
    assert np.allclose(rr, ref.real, rtol=0, atol=1e-15) and np.allclose(ri, ref.imag, rtol=0, atol=1e-15)
    assert np.all(sr >= np.abs(rr)) and np.all(si >= np.abs(ri))


def test_mrifhd_fh_complex_exponential_closed_form():
    # rF + i iF = sum_k RhoPhi_k exp(i arg_k)  (complex arithmetic, not the real expansion)
    d = synth.mrifhd_inputs(4, 97, 5)
    rr, ri, _, _ = be.mrifhd_rhophi(d["phiR"], d["phiI"], d["dR"], d["dI"])
    rF, iF, Sr, Si = be.mrifhd_fh(d["x"], d["y"], d["z"], d["kx"], d["ky"], d["kz"], rr, ri)
    f64 = {k: v.astype(np.float64) for k, v in d.items()}
    arg = be.TWO_PI_F32 * (np.outer(f64["x"], f64["kx"]) + np.outer(f64["y"], f64["ky"]) + np.outer(f64["z"], f64["kz"]))
    ref = (np.exp(1j * arg) * (rr + 1j * ri)[None, :]).sum(axis=1)
    assert np.max(np.abs(rF - ref.real) / Sr) < 1e-12 and np.max(np.abs(iF - ref.imag) / Si) < 1e-12


def test_mrifhd_origin_voxel_and_real_rhophi_reduces_to_mriq():
    g = np.random.default_rng(9)
    kx, ky, kz = (g.uniform(-8, 8, 40) for _ in range(3))
    rr, ri = g.uniform(-1, 1, 40), g.uniform(-1, 1, 40)
    zero = np.zeros(1)
    rF, iF, _, _ = be.mrifhd_fh(zero, zero, zero, kx, ky, kz, rr, ri)     # arg = 0: sums of RhoPhi
    assert abs(rF[0] - rr.sum()) < 1e-12 and abs(iF[0] - ri.sum()) < 1e-12
    # iRhoPhi = 0: (rFhD, iFhD) is mri-q's (Qr, Qi) with phiMag = rRhoPhi (mri-q is pinned above)
    d = synth.mriq_inputs(4, 40, 2)
    rF, iF, _, _ = be.mrifhd_fh(d["x"], d["y"], d["z"], kx, ky, kz, rr, np.zeros(40))
    qr, qi, _, _ = be.mriq_q(d["x"], d["y"], d["z"], kx, ky, kz, rr)
    assert np.allclose(rF, qr, rtol=0, atol=1e-12) and np.allclose(iF, qi, rtol=0, atol=1e-12)


def test_mrifhd_chunks_accumulate():
    d = synth.mrifhd_inputs(4, 64, 1)
    rr, ri, _, _ = be.mrifhd_rhophi(d["phiR"], d["phiI"], d["dR"], d["dI"])
    args = (d["x"], d["y"], d["z"])
    full = be.mrifhd_fh(*args, d["kx"], d["ky"], d["kz"], rr, ri)
    a = be.mrifhd_fh(*args, d["kx"][:30], d["ky"][:30], d["kz"][:30], rr[:30], ri[:30])
    b = be.mrifhd_fh(*args, d["kx"][30:], d["ky"][30:], d["kz"][30:], rr[30:], ri[30:], a[0], a[1])
    assert np.allclose(b[0], full[0], rtol=0, atol=1e-12) and np.allclose(b[1], full[1], rtol=0, atol=1e-12)


# ------------------------------------------------------------------ NEXT-3 cp (reading 14)
def test_cp_single_atom_closed_form():
    # q = 2 at (0, 0, z + 1), h = 1: V(0,0) = 2/1, V(3,4) = 2/sqrt(9 + 16 + 1)
    z = 5.0
    V, S = be.cp(np.array([[0.0, 0.0, z + 1.0, 2.0]]), 6, 6, 1.0, z)
    assert V[0] == 2.0
    assert abs(V[4 * 6 + 3] - 2.0 / math.sqrt(26.0)) < 1e-15
    assert np.array_equal(np.abs(V), S)


def test_cp_bruteforce_loops_linearity_accumulate():
    at, z = synth.cp_inputs(13, 5, 4, 0.7, seed=3)
    V, S = be.cp(at, 5, 4, 0.7, z)
    for j in range(4):
        for i in range(5):
            e = 0.0
            for a in at.astype(np.float64):
                e += a[3] / math.sqrt((i * 0.7 - a[0]) ** 2 + (j * 0.7 - a[1]) ** 2 + (z - a[2]) ** 2)
            assert abs(V[j * 5 + i] - e) <= 1e-12 * S[j * 5 + i]
    # linearity in the charges and accumulation over atom chunks
    at2 = at.astype(np.float64)
    at2[:, 3] *= -3.0
    V2, _ = be.cp(at2, 5, 4, 0.7, z)
    assert np.allclose(V2, -3.0 * V, rtol=1e-12, atol=0)
    Va, _ = be.cp(at[:6], 5, 4, 0.7, z)
    Vb, _ = be.cp(at[6:], 5, 4, 0.7, z, V_in=Va)
    assert np.allclose(Vb, V, rtol=1e-12, atol=0)


# ------------------------------------------------------------------ NEXT-3 fft (reading 15)
def test_fft_matches_library_fft():
    # second opinion: numpy's FFT (a different algorithm) on a ragged batch of several lengths
    for n in (2, 8, 64, 256):
        x = synth.fft_inputs(5, n, seed=n)
        xc = x[..., 0].astype(np.float64) + 1j * x[..., 1]
        X, S = be.fft(xc)
        assert np.max(np.abs(X - np.fft.fft(xc, axis=-1)) / S) < 1e-13


def test_fft_bruteforce_loops():
    x = synth.fft_inputs(2, 8, seed=3)
    xc = x[..., 0].astype(np.float64) + 1j * x[..., 1]
    X, _ = be.fft(xc)
    for b in range(2):
        for k in range(8):
            s = sum(complex(xc[b, j]) * cmath.exp(-2j * math.pi * j * k / 8) for j in range(8))
            assert abs(X[b, k] - s) < 1e-13


def test_fft_closed_forms():
    n = 64
    # impulse at m -> X[k] = exp(-2 pi i m k / n); tone m -> n delta_{k, m}; constant -> n c delta_k0
    imp = synth.fft_inputs(n, n, 0, "impulse")
    X, _ = be.fft(imp[..., 0] + 1j * imp[..., 1])
    m, k = np.meshgrid(np.arange(n), np.arange(n), indexing="ij")
    assert np.max(np.abs(X - np.exp(-2j * np.pi * m * k / n))) < 1e-13
    tone = synth.fft_inputs(n, n, 0, "tone").astype(np.float64)
    X, _ = be.fft(tone[..., 0] + 1j * tone[..., 1])
    assert np.max(np.abs(X - n * np.eye(n))) < 1e-4            # the tone itself is fp32-rounded
    X, S = be.fft(np.full((1, n), 0.25 - 0.5j))
    assert abs(X[0, 0] - n * (0.25 - 0.5j)) < 1e-13 and np.max(np.abs(X[0, 1:])) < 1e-13
    assert np.allclose(S, n * abs(0.25 - 0.5j))


def test_fft_parseval_linearity_shift():
    n = 128
    x = synth.fft_inputs(3, n, seed=11)
    xc = x[..., 0].astype(np.float64) + 1j * x[..., 1]
    X, _ = be.fft(xc)
    assert np.allclose((np.abs(X) ** 2).sum(-1), n * (np.abs(xc) ** 2).sum(-1), rtol=1e-12)
    Y, _ = be.fft(2.5 * xc + 1j * xc[::-1])
    assert np.allclose(Y, 2.5 * X + 1j * X[::-1], rtol=0, atol=1e-11)
    Z, _ = be.fft(np.roll(xc, 3, axis=-1))                      # x[j - 3] -> X[k] exp(-2 pi i 3 k / n)
    assert np.allclose(Z, X * np.exp(-2j * np.pi * 3 * np.arange(n) / n), rtol=0, atol=1e-11)


# ------------------------------------------------------------------ NEXT-3 tpacf (reading 16)
def test_tpacf_bruteforce_loops():
    e = synth.tpacf_edges()
    A = synth.tpacf_inputs(40, 1)
    B = synth.tpacf_inputs(23, 2)
    f = np.float32
    for self_pairs, X, Y in ((True, A, A), (False, A, B)):
        cnt = [0] * (len(e) + 1)
        for i in range(X.shape[0]):
            for j in range(Y.shape[0]):
                if self_pairs and j <= i:
                    continue
                d = f(f(f(X[i, 0]) * f(Y[j, 0])) + f(f(X[i, 1]) * f(Y[j, 1])))
                d = f(d + f(f(X[i, 2]) * f(Y[j, 2])))
                b = 0
                for k in range(len(e)):
                    if d < e[k]:
                        b += 1
                cnt[b] += 1
        assert list(be.tpacf(X, Y, e, self_pairs)) == cnt


def test_tpacf_counts_and_exact_geometry():
    e = synth.tpacf_edges()
    nb = len(e) + 1
    A = synth.tpacf_inputs(700, 5)
    B = synth.tpacf_inputs(300, 6, "uniform")
    assert be.tpacf(A, A, e, True).sum() == 700 * 699 // 2
    assert be.tpacf(A, B, e, False).sum() == 700 * 300
    # cross is symmetric; cross(A, A) = 2 self(A) + the i == j pairs
    assert np.array_equal(be.tpacf(A, B, e, False), be.tpacf(B, A, e, False))
    diag = np.bincount(be.tpacf_bin(be.tpacf_dot_f32(A, A), e), minlength=nb)
    assert np.array_equal(be.tpacf(A, A, e, False), 2 * be.tpacf(A, A, e, True) + diag)
    # axis points: identical -> dot 1 (bin 0), orthogonal -> dot 0, antipodal -> dot -1 (last bin)
    ax = np.array([[1, 0, 0], [0, 1, 0], [-1, 0, 0]], np.float32)
    c = be.tpacf(ax[:1], ax, e, False)
    assert c[0] == 1 and c[nb - 1] == 1 and c[int((e > 0).sum())] == 1
