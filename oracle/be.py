"""BE (CUDA-core) kernels, fp64 / exact-integer reference.  Test infrastructure only.

The paper uses the Parboil suite as BE applications (Table II) and
gives no definitions of the kernels; BASELINE.json adds spmv, histo and bfs.  Each
function below writes out the plain definition in the reading recorded in DESIGN.md §2
(= SURVEY.md §8(c) rows c3-c10), and returns the exact value plus, for floating point,
the absolute sum of the terms (for metrics.rel_err).
"""
from __future__ import annotations

import math
from collections import deque

import numpy as np

# ----------------------------------------------------------------------------- c3 sgemm
def sgemm(A, B, alpha=1.0, beta=0.0, C_in=None):
    """C = alpha * A.B + beta * C_in, row-major A [M,K], B [K,N] (Parboil sgemm).

    Reading: Parboil's column-major "NT" form is the same math on transposed storage;
    alpha=1, beta=0 at the BASELINE configs.
    """
    A64 = np.asarray(A, np.float64)
    B64 = np.asarray(B, np.float64)
    C = alpha * (A64 @ B64)
    S = abs(alpha) * (np.abs(A64) @ np.abs(B64))
    if beta != 0.0:
        c = np.asarray(C_in, np.float64)
        C = C + beta * c
        S = S + abs(beta) * np.abs(c)
    return C, S


# ----------------------------------------------------------------------------- c4 stencil
def stencil(A0, c0, c1):
    """One 7-point Jacobi sweep (Parboil stencil):

        An[z,y,x] = c1*(A[z,y,x-1]+A[z,y,x+1]+A[z,y-1,x]+A[z,y+1,x]+A[z-1,y,x]+A[z+1,y,x])
                    - c0*A[z,y,x]      for interior cells,
        An = A                          on the boundary (Parboil copies both buffers).

    A0 is [nz][ny][nx] with x fastest.
    """
    A = np.asarray(A0, np.float64)
    An = A.copy()
    S = np.abs(A).copy()
    if min(A.shape) < 3:
        return An, S
    c = A[1:-1, 1:-1, 1:-1]
    nb = (A[1:-1, 1:-1, :-2] + A[1:-1, 1:-1, 2:] + A[1:-1, :-2, 1:-1] + A[1:-1, 2:, 1:-1]
          + A[:-2, 1:-1, 1:-1] + A[2:, 1:-1, 1:-1])
    nba = (np.abs(A[1:-1, 1:-1, :-2]) + np.abs(A[1:-1, 1:-1, 2:]) + np.abs(A[1:-1, :-2, 1:-1])
           + np.abs(A[1:-1, 2:, 1:-1]) + np.abs(A[:-2, 1:-1, 1:-1]) + np.abs(A[2:, 1:-1, 1:-1]))
    An[1:-1, 1:-1, 1:-1] = float(c1) * nb - float(c0) * c
    S[1:-1, 1:-1, 1:-1] = abs(float(c1)) * nba + abs(float(c0)) * np.abs(c)
    return An, S


# ----------------------------------------------------------------------------- c5 mri-q
TWO_PI_F32 = float(np.float32(6.2831853071795864769))  # Parboil's PIx2 constant as fp32


def mriq_phimag(phiR, phiI):
    """ComputePhiMag: phiMag[k] = phiR[k]^2 + phiI[k]^2 (Parboil mri-q)."""
    r = np.asarray(phiR, np.float64)
    i = np.asarray(phiI, np.float64)
    return r * r + i * i, r * r + i * i


def mriq_q(x, y, z, kx, ky, kz, phiMag, Qr_in=None, Qi_in=None):
    """ComputeQ over one k chunk (accumulating into Qr_in/Qi_in when given):

        Qr[v] += sum_k phiMag[k] * cos(2*pi*(kx[k]*x[v] + ky[k]*y[v] + kz[k]*z[v]))
        Qi[v] += sum_k phiMag[k] * sin(2*pi*(...))

    fp64 throughout with 2*pi = Parboil's PIx2 rounded to fp32 (the constant both sides use).
    """
    x, y, z = (np.asarray(a, np.float64) for a in (x, y, z))
    nv = x.size
    Qr = np.zeros(nv) if Qr_in is None else np.asarray(Qr_in, np.float64).copy()
    Qi = np.zeros(nv) if Qi_in is None else np.asarray(Qi_in, np.float64).copy()
    Sr = np.abs(Qr).copy()
    Si = np.abs(Qi).copy()
    kx, ky, kz, pm = (np.asarray(a, np.float64) for a in (kx, ky, kz, phiMag))
    step = 256
    for k0 in range(0, kx.size, step):
        arg = TWO_PI_F32 * (np.outer(x, kx[k0:k0 + step]) + np.outer(y, ky[k0:k0 + step])
                            + np.outer(z, kz[k0:k0 + step]))
        c = np.cos(arg) * pm[None, k0:k0 + step]
        s = np.sin(arg) * pm[None, k0:k0 + step]
        Qr += c.sum(axis=1)
        Qi += s.sum(axis=1)
        Sr += np.abs(c).sum(axis=1)
        Si += np.abs(s).sum(axis=1)
    return Qr, Qi, Sr, Si


# ----------------------------------------------------------------------------- NEXT-3 mri-fhd
def mrifhd_rhophi(phiR, phiI, dR, dI):
    """ComputeRhoPhi (Parboil mri-fhd, Table II; not defined in the paper, DESIGN.md
    §2 reading 14): rRhoPhi = phiR*dR + phiI*dI, iRhoPhi = phiR*dI - phiI*dR.  Returns
    (rRhoPhi, iRhoPhi, abs-sum of the r terms, abs-sum of the i terms)."""
    pr, pi, r, i = (np.asarray(a, np.float64) for a in (phiR, phiI, dR, dI))
    return pr * r + pi * i, pr * i - pi * r, np.abs(pr * r) + np.abs(pi * i), np.abs(pr * i) + np.abs(pi * r)


def mrifhd_fh(x, y, z, kx, ky, kz, rRhoPhi, iRhoPhi, rF_in=None, iF_in=None):
    """ComputeFH over one k chunk (accumulating into rF_in / iF_in when given):

        arg = 2*pi*(kx[k]*x[v] + ky[k]*y[v] + kz[k]*z[v])
        rFhD[v] += sum_k rRhoPhi[k]*cos(arg) - iRhoPhi[k]*sin(arg)
        iFhD[v] += sum_k iRhoPhi[k]*cos(arg) + rRhoPhi[k]*sin(arg)

    fp64 with 2*pi = Parboil's fp32 PIx2 (as mri-q).  Returns (rFhD, iFhD, Sr, Si), S = abs-sums."""
    x, y, z = (np.asarray(a, np.float64) for a in (x, y, z))
    nv = x.size
    rF = np.zeros(nv) if rF_in is None else np.asarray(rF_in, np.float64).copy()
    iF = np.zeros(nv) if iF_in is None else np.asarray(iF_in, np.float64).copy()
    Sr, Si = np.abs(rF).copy(), np.abs(iF).copy()
    kx, ky, kz, rr, ri = (np.asarray(a, np.float64) for a in (kx, ky, kz, rRhoPhi, iRhoPhi))
    step = 256
    for k0 in range(0, kx.size, step):
        sl = slice(k0, k0 + step)
        arg = TWO_PI_F32 * (np.outer(x, kx[sl]) + np.outer(y, ky[sl]) + np.outer(z, kz[sl]))
        c, s_ = np.cos(arg), np.sin(arg)
        t1, t2 = c * rr[None, sl], s_ * ri[None, sl]      # rF terms
        t3, t4 = c * ri[None, sl], s_ * rr[None, sl]      # iF terms
        rF += (t1 - t2).sum(axis=1)
        iF += (t3 + t4).sum(axis=1)
        Sr += (np.abs(t1) + np.abs(t2)).sum(axis=1)
        Si += (np.abs(t3) + np.abs(t4)).sum(axis=1)
    return rF, iF, Sr, Si


# ----------------------------------------------------------------------------- NEXT-3 cp
def cp(atoms, nx, ny, h, z, V_in=None):
    """Direct Coulomb summation on one lattice slice (Parboil cp, Table II; not
    defined in the paper, DESIGN.md §2 reading 14), accumulating into V_in when given:

        V[j, i] += sum_a q_a / sqrt((i*h - x_a)^2 + (j*h - y_a)^2 + (z - z_a)^2)

    lattice point (i, j) at (i*h, j*h, z), flat index j*nx + i.  Returns (V, abs-sum)."""
    at = np.asarray(atoms, np.float64)
    px = np.arange(nx, dtype=np.float64) * h
    py = np.arange(ny, dtype=np.float64) * h
    V = np.zeros(ny * nx) if V_in is None else np.asarray(V_in, np.float64).ravel().copy()
    S = np.abs(V).copy()
    gx, gy = np.meshgrid(px, py)                 # [ny, nx]
    gx, gy = gx.ravel(), gy.ravel()
    for a in range(at.shape[0]):
        ax, ay, az, q = at[a]
        e = q / np.sqrt((gx - ax) ** 2 + (gy - ay) ** 2 + (z - az) ** 2)
        V += e
        S += np.abs(e)
    return V, S


# ----------------------------------------------------------------------------- c6 cutcp
CUTCP_CUTOFF = 12.0
CUTCP_EXCL = 1.0


def cutcp(atoms, nx, ny, nz, h, cutoff=CUTCP_CUTOFF, excl=CUTCP_EXCL, points=None):
    """Cutoff Coulomb potential on a lattice (Parboil cutcp):

        V[p] = sum_{a : d^2 < c^2} q_a / d * (1 - d^2/c^2)^2,   d = |p - r_a|,
        V[p] = 0 if any atom has d < excl (exclusion),
    lattice point (i,j,k) at (i*h, j*h, k*h), flat index (k*ny + j)*nx + i.
    Brute force over all atoms; `points` optionally restricts to flat indices.
    """
    at = np.asarray(atoms, np.float64)
    pos, q = at[:, :3], at[:, 3]
    if points is None:
        points = np.arange(nx * ny * nz)
    points = np.asarray(points)
    V = np.zeros(points.size)
    S = np.zeros(points.size)
    c2 = cutoff * cutoff
    for n, f in enumerate(points):
        i = f % nx
        j = (f // nx) % ny
        k = f // (nx * ny)
        p = np.array([i * h, j * h, k * h], np.float64)
        d2 = ((pos - p) ** 2).sum(axis=1)
        if np.any(d2 < excl * excl):
            continue
        m = d2 < c2
        s = (1.0 - d2[m] / c2)
        e = q[m] / np.sqrt(d2[m]) * s * s
        V[n] = e.sum()
        S[n] = np.abs(e).sum()
    return V, S


def cutcp_bins(atoms, bdim, bin_size, depth):
    """Atom binning feeding the GPU cutcp (a data layout): bin
    b = (floor(z/bs)*by + floor(y/bs))*bx + floor(x/bs), clamped into the grid, holds its atoms
    in atom-index order; unused slots (1e30, 1e30, 1e30, 0).  Returns (bins, count)."""
    bx, by, bz = bdim
    at = np.asarray(atoms, np.float32)
    bins = np.tile(np.array([1e30, 1e30, 1e30, 0.0], np.float32), (bx * by * bz, depth, 1))
    count = np.zeros(bx * by * bz, np.int64)
    for a in range(at.shape[0]):
        ix = min(max(int(np.floor(at[a, 0] / bin_size)), 0), bx - 1)
        iy = min(max(int(np.floor(at[a, 1] / bin_size)), 0), by - 1)
        iz = min(max(int(np.floor(at[a, 2] / bin_size)), 0), bz - 1)
        b = (iz * by + iy) * bx + ix
        if count[b] < depth:
            bins[b, count[b]] = at[a]
        count[b] += 1
    return bins, count


# ----------------------------------------------------------------------------- c7 lbm
import synth as _synth  # direction table only (data, not arithmetic)

LBM_E = np.array([[d[1], d[2], d[3]] for d in _synth.LBM_DIRS], np.int64)
LBM_W = np.array([1 / 3] + [1 / 18] * 6 + [1 / 36] * 12, np.float64)
LBM_OMEGA = 1.95
LBM_ACCEL_U = (0.005, 0.002, 0.0)


def lbm_opposite(i: int) -> int:
    e = LBM_E[i]
    for j in range(19):
        if np.all(LBM_E[j] == -e):
            return j
    raise AssertionError


def lbm_step(src, flags, dst_init):
    """One D3Q19 BGK stream-collide step, push form (Parboil lbm), reading per
    DESIGN.md §2:
      OBSTACLE cell x: dst_{opp(i)}[x + e_opp(i)] = src_i[x]    (full-way bounce back)
      otherwise: rho = sum f_i, u = sum f_i e_i / rho; ACCEL cells use u = (0.005,0.002,0);
        feq_i = w_i rho (1 + 3 e_i.u + 4.5 (e_i.u)^2 - 1.5 u.u)
        dst_i[x + e_i] = (1-omega) f_i + omega feq_i
    Pushes whose destination lies outside the grid are discarded; entries never written keep
    dst_init.  src/dst are [19][nz][ny][nx]; flags [nz][ny][nx].
    """
    f = np.asarray(src, np.float64)
    fl = np.asarray(flags)
    nz, ny, nx = fl.shape
    dst = np.asarray(dst_init, np.float64).copy()
    S = np.abs(dst).copy()
    rho = f.sum(axis=0)
    u = np.stack([(f * LBM_E[:, a, None, None, None]).sum(axis=0) for a in range(3)]) / rho
    acc = fl == _synth.LBM_ACCEL
    for a in range(3):
        u[a][acc] = LBM_ACCEL_U[a]
    u2 = (u * u).sum(axis=0)
    obst = fl == _synth.LBM_OBSTACLE
    for i in range(19):
        eu = LBM_E[i, 0] * u[0] + LBM_E[i, 1] * u[1] + LBM_E[i, 2] * u[2]
        feq = LBM_W[i] * rho * (1.0 + 3.0 * eu + 4.5 * eu * eu - 1.5 * u2)
        feqa = LBM_W[i] * rho * (1.0 + 3.0 * np.abs(eu) + 4.5 * eu * eu + 1.5 * u2)
        val = (1.0 - LBM_OMEGA) * f[i] + LBM_OMEGA * feq
        vabs = abs(1.0 - LBM_OMEGA) * np.abs(f[i]) + LBM_OMEGA * feqa
        # obstacle cells: reflected copy of the unrelaxed value into the opposite slot
        j = lbm_opposite(i)
        ex, ey, ez = LBM_E[j]
        for (m, v, va, slot, (dx, dy, dz)) in ((~obst, val, vabs, i, LBM_E[i]),
                                                (obst, f[i], np.abs(f[i]), j, (ex, ey, ez))):
            zs, ys, xs = np.nonzero(m)
            tz, ty, tx = zs + dz, ys + dy, xs + dx
            ok = (tz >= 0) & (tz < nz) & (ty >= 0) & (ty < ny) & (tx >= 0) & (tx < nx)
            dst[slot, tz[ok], ty[ok], tx[ok]] = v[zs[ok], ys[ok], xs[ok]]
            S[slot, tz[ok], ty[ok], tx[ok]] = va[zs[ok], ys[ok], xs[ok]]
    return dst, S


def lbm_written_mask(nx, ny, nz):
    """True where lbm_step writes dst_i[x]: the upstream cell x - e_i lies inside the grid."""
    m = np.zeros((19, nz, ny, nx), bool)
    for i in range(19):
        dx, dy, dz = LBM_E[i]
        m[i, max(dz, 0):nz + min(dz, 0), max(dy, 0):ny + min(dy, 0), max(dx, 0):nx + min(dx, 0)] = True
    return m


# ----------------------------------------------------------------------------- c8 spmv (JDS)
def jds_build(row_ptr, cols, vals):
    """CSR -> JDS (Parboil spmv format), reading per DESIGN.md §2:
      perm     rows sorted by length descending, ties by row index ascending (stable)
      row_len  len[perm[i]]
      jds_ptr  jds_ptr[d] = start of jagged diagonal d; jds_ptr[d+1]-jds_ptr[d] = #{r : len_r > d}
      jds_col/jds_val: element (d, i) = d-th nonzero of row perm[i], at jds_ptr[d] + i.
    """
    row_ptr = np.asarray(row_ptr, np.int64)
    R = row_ptr.size - 1
    lens = [int(row_ptr[r + 1] - row_ptr[r]) for r in range(R)]
    perm = sorted(range(R), key=lambda r: (-lens[r], r))
    maxlen = lens[perm[0]] if R else 0
    jds_ptr = [0]
    for d in range(maxlen):
        jds_ptr.append(jds_ptr[-1] + sum(1 for L in lens if L > d))
    nnz = jds_ptr[-1]
    jcol = np.zeros(nnz, np.int32)
    jval = np.zeros(nnz, np.float32)
    for i, r in enumerate(perm):
        for d in range(lens[r]):
            jcol[jds_ptr[d] + i] = cols[row_ptr[r] + d]
            jval[jds_ptr[d] + i] = vals[row_ptr[r] + d]
    return (np.array(perm, np.int32), np.array([lens[r] for r in perm], np.int32),
            np.array(jds_ptr, np.int32), jcol, jval)


def spmv_jds(perm, row_len, jds_ptr, jcol, jval, x):
    """y[perm[i]] = sum_{d < row_len[i]} jval[jds_ptr[d]+i] * x[jcol[jds_ptr[d]+i]] (fp64)."""
    x64 = np.asarray(x, np.float64)
    R = len(perm)
    y = np.zeros(R)
    S = np.zeros(R)
    for i in range(R):
        idx = np.asarray(jds_ptr[:row_len[i]], np.int64) + i
        t = np.asarray(jval, np.float64)[idx] * x64[np.asarray(jcol)[idx]]
        y[perm[i]] = t.sum()
        S[perm[i]] = np.abs(t).sum()
    return y, S


def spmv_csr(row_ptr, cols, vals, x):
    """Second opinion: y = A x straight from CSR."""
    x64 = np.asarray(x, np.float64)
    R = len(row_ptr) - 1
    y = np.zeros(R)
    for r in range(R):
        a, b = row_ptr[r], row_ptr[r + 1]
        y[r] = float((np.asarray(vals[a:b], np.float64) * x64[cols[a:b]]).sum())
    return y


# ----------------------------------------------------------------------------- c9 histo
def histo(values, nbins):
    """count[b] = #{i : values[i] == b} (u32), values assumed < nbins (Parboil-style histo)."""
    cnt = np.zeros(nbins, np.int64)
    v = np.asarray(values, np.int64)
    np.add.at(cnt, v, 1)
    return cnt.astype(np.uint32)


def histo_saturate(count):
    """Parboil u8 view: sat[b] = min(count[b], 255)."""
    return np.minimum(np.asarray(count, np.int64), 255).astype(np.uint8)


# ----------------------------------------------------------------------------- c10 bfs
def bfs_levels(row_ptr, col, src=0):
    """Textbook queue BFS: level[v] = hop distance from src, -1 if unreachable."""
    V = len(row_ptr) - 1
    level = np.full(V, -1, np.int32)
    level[src] = 0
    dq = deque([src])
    while dq:
        v = dq.popleft()
        for e in range(row_ptr[v], row_ptr[v + 1]):
            u = col[e]
            if level[u] < 0:
                level[u] = level[v] + 1
                dq.append(u)
    return level


def bfs_expand(row_ptr, col, level, mask, visited, upd):
    """Rodinia Kernel1: for v with mask[v]: clear mask[v]; for each neighbour u with
    !visited[u]: level[u] = level[v] + 1, upd[u] = 1.  Returns new (level, mask, upd)."""
    level = np.array(level, np.int32)
    mask = np.array(mask, np.uint8)
    upd = np.array(upd, np.uint8)
    front = np.nonzero(mask)[0]
    for v in front:
        mask[v] = 0
        for e in range(row_ptr[v], row_ptr[v + 1]):
            u = col[e]
            if not visited[u]:
                level[u] = level[v] + 1
                upd[u] = 1
    return level, mask, upd


def bfs_commit(mask, visited, upd):
    """Rodinia Kernel2: for u with upd[u]: mask[u] = visited[u] = 1, upd[u] = 0; over = any."""
    mask = np.array(mask, np.uint8)
    visited = np.array(visited, np.uint8)
    upd = np.array(upd, np.uint8)
    idx = np.nonzero(upd)[0]
    mask[idx] = 1
    visited[idx] = 1
    upd[idx] = 0
    return mask, visited, upd, int(idx.size > 0)


# ----------------------------------------------------------------------------- fma_burn (Kc)
def fma_burn(n_threads, iters, a=0.5, b_scale=0.125):
    """Register-only FMA micro-kernel "Kc" (§III-B): thread g runs 4 independent
    recurrences x_j <- x_j * a + b_j with x_j(0) = (g % 97 + j) / 128, b_j = b_scale*(j+1),
    and outputs ((x_0 + x_1) + x_2) + x_3.  fp64 here; the kernel's fp32 rounding error is
    contracted by |a| = 1/2 each step, so it stays within a few ulp (bound 2 ulp/step sum)."""
    g = np.arange(n_threads, dtype=np.float64)
    out = np.zeros(n_threads)
    for j in range(4):
        x = (np.mod(g, 97) + j) / 128.0
        bj = b_scale * (j + 1)
        # closed form of the affine recurrence x_n = a^n x_0 + b (1 - a^n) / (1 - a)
        an = a ** iters
        out += an * x + bj * (1.0 - an) / (1.0 - a)
    return out


# ----------------------------------------------------------------------------- NEXT-3 fft
def fft(x):
    """Batched forward complex DFT (Parboil fft, Table II; the GEMM-fft pair of Fig. 10
    P:1417-1419; not defined in the paper, DESIGN.md §2 reading 15), written out as the definition:

        X[b, k] = sum_j x[b, j] * exp(-2 pi i (j k mod n) / n),   0 <= j, k < n

    x: complex [batch, n].  fp64 (complex128) with the twiddle of each (j k mod n) evaluated by
    numpy's exp.  Returns (X, S) with S[b, k] = sum_j |x[b, j]| (every term has modulus |x[b, j]|;
    the abs-sum of metrics.max_rel_err for both the real and the imaginary part)."""
    x = np.asarray(x, np.complex128)
    n = x.shape[-1]
    jk = np.mod(np.outer(np.arange(n), np.arange(n)), n)
    W = np.exp(-2j * np.pi * jk / n)
    X = x @ W
    S = np.repeat(np.abs(x).sum(axis=-1, keepdims=True), n, axis=-1)
    return X, S


# ----------------------------------------------------------------------------- NEXT-3 tpacf
def tpacf_dot_f32(a, b):
    """The pair's cosine as the kernel computes it, in fp32 with every product and sum rounded
    (no FMA): ((ax*bx + ay*by) + az*bz).  Integer counts are decided from this value, so both
    sides take the decision in the same precision (DESIGN.md §2 reading 16)."""
    a = np.asarray(a, np.float32)
    b = np.asarray(b, np.float32)
    return ((a[..., 0] * b[..., 0]) + (a[..., 1] * b[..., 1])) + (a[..., 2] * b[..., 2])


def tpacf_bin(dot, edges):
    """bin(dot) = #{k : dot < edges[k]} for the strictly decreasing fp32 cosines of increasing
    angular bin edges: 0 = closer than edges[0], len(edges) = wider than the last edge."""
    dot = np.asarray(dot, np.float32)
    e = np.asarray(edges, np.float32)
    return (dot[..., None] < e).sum(axis=-1)


def tpacf(A, B, edges, self_pairs):
    """Two-point angular correlation histogram (Parboil tpacf, Table II; reading 16):

        count[b] = #{pairs (i, j) : bin(dot_f32(A[i], B[j])) == b},  b in [0, len(edges)]

    over all pairs i, j (cross correlation, DR) or over i < j with B = A (self correlation, DD /
    RR when self_pairs).  A, B: unit vectors float32 [n, 3].  Returns int64 [len(edges) + 1]."""
    A = np.asarray(A, np.float32)
    B = np.asarray(B, np.float32)
    nb = len(edges) + 1
    cnt = np.zeros(nb, np.int64)
    step = 256
    for i0 in range(0, A.shape[0], step):
        a = A[i0:i0 + step]
        bins = tpacf_bin(tpacf_dot_f32(a[:, None, :], B[None, :, :]), edges)
        if self_pairs:
            ii = np.arange(i0, i0 + a.shape[0])[:, None]
            jj = np.arange(B.shape[0])[None, :]
            bins = bins[jj > ii]
        cnt += np.bincount(bins.ravel(), minlength=nb)
    return cnt
