"""Seeded synthetic input generators shared by the CPU oracle and the GPU harness.

This module holds NO arithmetic of the method (no GEMM, conv, stencil, ...): it only
draws seeded random inputs with the shapes, value distributions and structure of
the paper's workloads, following the recipe in DESIGN.md §3 (= SURVEY.md §8(c).2).
Both `oracle/` and the product tests/bench import it; neither imports the other.

RNG: numpy.random.Generator(PCG64(seed)).  fp16 arrays are drawn as fp32 and
rounded with .astype(float16) (round-to-nearest-even).  Everything C-contiguous.

Workload shape tables (ResNet-50 / VGG-16 batch-1 convolutions, BERT-base seq-128
GEMMs) describe the LC services of BASELINE.json configs 2-4; the paper's LC
services are ResNet50 and VGG16 (Table II).
"""
from __future__ import annotations

import math
from dataclasses import dataclass

import numpy as np


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


# --------------------------------------------------------------------------- LC GEMM
def lc_gemm_inputs(M: int, N: int, K: int, seed: int, variant: str = "uniform"):
    """A [M,K] fp16 K-major, B [N,K] fp16 K-major ("TN").  D = A . B^T.

    variant: "uniform" U[-1,1); "int" uniform in {-4..4}; "identity" B = I (N==K);
    "onehot" each row of A has a single 1.0 at a uniform column, B uniform.
    """
    g = rng(seed)
    if variant == "int":
        A = g.integers(-4, 5, size=(M, K)).astype(np.float16)
        B = g.integers(-4, 5, size=(N, K)).astype(np.float16)
    else:
        A = g.uniform(-1.0, 1.0, size=(M, K)).astype(np.float32).astype(np.float16)
        B = g.uniform(-1.0, 1.0, size=(N, K)).astype(np.float32).astype(np.float16)
        if variant == "identity":
            assert N == K
            B = np.eye(N, dtype=np.float16)
        elif variant == "onehot":
            A = np.zeros((M, K), np.float16)
            A[np.arange(M), g.integers(0, K, size=M)] = 1.0
        elif variant != "uniform":
            raise ValueError(variant)
    return np.ascontiguousarray(A), np.ascontiguousarray(B)


# --------------------------------------------------------------------------- LC conv
@dataclass(frozen=True)
class ConvShape:
    name: str
    n: int
    h: int
    w: int
    c: int
    k: int
    r: int
    s: int
    stride: int
    pad: int

    @property
    def p(self) -> int:
        return (self.h + 2 * self.pad - self.r) // self.stride + 1

    @property
    def q(self) -> int:
        return (self.w + 2 * self.pad - self.s) // self.stride + 1

    @property
    def gemm_mnk(self):
        return self.n * self.p * self.q, self.k, self.c * self.r * self.s

    @property
    def flops(self) -> int:
        M, N, K = self.gemm_mnk
        return 2 * M * N * K


def resnet50_convs(batch: int = 1) -> list[ConvShape]:
    """The 53 convolutions of ResNet-50 v1.5 at 224x224 (stride on the 3x3).

    conv1's C=3 input is zero-padded to C=8 channels so that the NHWC row pitch is
    a multiple of 16 bytes (TMA); zero channels do not change the result.
    """
    out = [ConvShape("conv1", batch, 224, 224, 8, 64, 7, 7, 2, 3)]
    cin, hw = 64, 56
    for li, (blocks, mid, cout) in enumerate([(3, 64, 256), (4, 128, 512), (6, 256, 1024), (3, 512, 2048)]):
        for b in range(blocks):
            stride = 2 if (b == 0 and li > 0) else 1
            hin = hw
            hout = hin // stride
            pre = f"layer{li + 1}.{b}"
            out.append(ConvShape(pre + ".conv1", batch, hin, hin, cin, mid, 1, 1, 1, 0))
            out.append(ConvShape(pre + ".conv2", batch, hin, hin, mid, mid, 3, 3, stride, 1))
            out.append(ConvShape(pre + ".conv3", batch, hout, hout, mid, cout, 1, 1, 1, 0))
            if b == 0:
                out.append(ConvShape(pre + ".downsample", batch, hin, hin, cin, cout, 1, 1, stride, 0))
            cin, hw = cout, hout
    assert len(out) == 53
    return out


def vgg16_convs(batch: int = 1) -> list[ConvShape]:
    cfg = [(64, 224), (64, 224), (128, 112), (128, 112), (256, 56), (256, 56), (256, 56),
           (512, 28), (512, 28), (512, 28), (512, 14), (512, 14), (512, 14)]
    out, cin = [], 8  # conv1_1 input padded 3 -> 8 channels
    for i, (k, hw) in enumerate(cfg):
        out.append(ConvShape(f"conv{i}", batch, hw, hw, cin, k, 3, 3, 1, 1))
        cin = k
    return out


def bert_base_gemms(seq: int = 128):
    """(name, M, N, K) of one BERT-base encoder layer at batch 1 (BASELINE config 3)."""
    return [("qkv", seq, 2304, 768), ("o", seq, 768, 768), ("ffn1", seq, 3072, 768), ("ffn2", seq, 768, 3072)]


def conv_inputs(cs: ConvShape, seed: int, variant: str = "uniform", real_c: int | None = None):
    """x NHWC fp16 U[0,1); w KRSC fp16 U[-1,1)*(C*R*S)^-1/2.  Channels >= real_c are zero."""
    g = rng(seed)
    if variant == "int":
        x = g.integers(0, 4, size=(cs.n, cs.h, cs.w, cs.c)).astype(np.float16)
        w = g.integers(-2, 3, size=(cs.k, cs.r, cs.s, cs.c)).astype(np.float16)
    else:
        x = g.uniform(0.0, 1.0, size=(cs.n, cs.h, cs.w, cs.c)).astype(np.float32).astype(np.float16)
        sc = 1.0 / math.sqrt(cs.c * cs.r * cs.s)
        w = (g.uniform(-1.0, 1.0, size=(cs.k, cs.r, cs.s, cs.c)) * sc).astype(np.float32).astype(np.float16)
    if real_c is not None and real_c < cs.c:
        x[..., real_c:] = 0
        w[..., real_c:] = 0
    bias = g.uniform(-0.1, 0.1, size=cs.k).astype(np.float32)
    return np.ascontiguousarray(x), np.ascontiguousarray(w), bias


# --------------------------------------------------------------------------- BE inputs
def sgemm_inputs(M: int, N: int, K: int, seed: int, variant: str = "uniform"):
    """A [M,K], B [K,N] fp32 row-major, U[0,1) (non-negative: well conditioned)."""
    g = rng(seed)
    if variant == "int":
        A = g.integers(-8, 9, size=(M, K)).astype(np.float32)
        B = g.integers(-8, 9, size=(K, N)).astype(np.float32)
    else:
        A = g.uniform(0.0, 1.0, size=(M, K)).astype(np.float32)
        B = g.uniform(0.0, 1.0, size=(K, N)).astype(np.float32)
    return A, B


def stencil_inputs(nx: int, ny: int, nz: int, seed: int, variant: str = "uniform"):
    """A0 [nz][ny][nx] fp32, x fastest.  'dyadic': small integers {0..15}."""
    g = rng(seed)
    if variant == "dyadic":
        return g.integers(0, 16, size=(nz, ny, nx)).astype(np.float32)
    return g.uniform(0.0, 1.0, size=(nz, ny, nx)).astype(np.float32)


def mriq_inputs(N: int, numK: int, seed: int):
    """N^3 voxel grid x=(i-N/2)/N etc (x fastest); k ~ U[-N/2,N/2)^3; phiR, phiI ~ U[-1,1)."""
    g = rng(seed)
    ax = ((np.arange(N) - N // 2) / N).astype(np.float32)
    z, y, x = np.meshgrid(ax, ax, ax, indexing="ij")
    kx, ky, kz = (g.uniform(-N / 2, N / 2, size=numK).astype(np.float32) for _ in range(3))
    phiR = g.uniform(-1, 1, size=numK).astype(np.float32)
    phiI = g.uniform(-1, 1, size=numK).astype(np.float32)
    return dict(x=x.ravel().copy(), y=y.ravel().copy(), z=z.ravel().copy(),
                kx=kx, ky=ky, kz=kz, phiR=phiR, phiI=phiI)


def mrifhd_inputs(N: int, numK: int, seed: int):
    """mri-q's voxel grid and k-space trajectory plus the data samples dR, dI ~ U[-1,1)."""
    d = mriq_inputs(N, numK, seed)
    g = rng(seed + 7919)
    d["dR"] = g.uniform(-1, 1, size=numK).astype(np.float32)
    d["dI"] = g.uniform(-1, 1, size=numK).astype(np.float32)
    return d


def cp_inputs(natoms: int, nx: int, ny: int, h: float, seed: int, z: float | None = None):
    """Parboil cp-like: natoms atoms U[0, L)^3 over the lattice box L = max(nx, ny)*h (z range
    the same), charges U[-1, 1); the slice height z defaults to L/2.  Atoms within 1e-3 of a
    lattice point of the slice are re-drawn (the potential there would be a near-singularity;
    only coordinates are compared).  Returns (atoms float32 [natoms, 4], z)."""
    g = rng(seed)
    L = max(nx, ny) * h
    z = L / 2 if z is None else z
    at = np.empty((natoms, 4), np.float32)
    for a in range(natoms):
        while True:
            p = g.uniform(0, L, size=3)
            far_x = abs(p[0] / h - round(p[0] / h)) * h > 1e-3
            far_y = abs(p[1] / h - round(p[1] / h)) * h > 1e-3
            if abs(p[2] - z) > 1e-3 or far_x or far_y:
                break
        at[a, :3] = p
        at[a, 3] = g.uniform(-1, 1)
    return at, float(np.float32(z))


def cutcp_inputs(L: float, seed: int, h: float = 0.5, density: float = 0.1, excl: float = 1.0):
    """Water-like box of side L (Angstrom): round(density*L^3) atoms U[0,L)^3, charges cycle
    (-0.834, +0.417, +0.417); lattice origin 0, ceil(L/h) points per axis, spacing h.

    Atoms placing any lattice point within 1e-4 A of the exclusion radius are re-drawn, so
    the exclusion predicate (d < excl) is never a rounding tie.  This conditioning only
    compares coordinates; it computes no potential.
    """
    g = rng(seed)
    natoms = int(round(density * L ** 3))
    npts = int(math.ceil(L / h))
    pos = np.empty((natoms, 3), np.float32)
    for i in range(natoms):
        while True:
            p = g.uniform(0.0, L, size=3).astype(np.float32)
            # nearest lattice points within excl+margin along each axis
            lo = np.maximum(np.floor((p - excl - 1e-3) / h).astype(int), 0)
            hi = np.minimum(np.ceil((p + excl + 1e-3) / h).astype(int), npts - 1)
            gx = np.arange(lo[0], hi[0] + 1) * h
            gy = np.arange(lo[1], hi[1] + 1) * h
            gz = np.arange(lo[2], hi[2] + 1) * h
            d = np.sqrt((gx[:, None, None] - p[0]) ** 2 + (gy[None, :, None] - p[1]) ** 2 + (gz[None, None, :] - p[2]) ** 2)
            if d.size == 0 or np.min(np.abs(d - excl)) > 1e-4:
                break
        pos[i] = p
    q = np.array([-0.834, 0.417, 0.417], np.float32)[np.arange(natoms) % 3]
    atoms = np.concatenate([pos, q[:, None]], axis=1).astype(np.float32)  # float4 (x,y,z,q)
    return dict(atoms=np.ascontiguousarray(atoms), nx=npts, ny=npts, nz=npts, h=np.float32(h))


# D3Q19 direction table (Parboil lbm order), used by both sides as a data table.
LBM_DIRS = [("C", 0, 0, 0), ("N", 0, 1, 0), ("S", 0, -1, 0), ("E", 1, 0, 0), ("W", -1, 0, 0),
            ("T", 0, 0, 1), ("B", 0, 0, -1), ("NE", 1, 1, 0), ("NW", -1, 1, 0), ("SE", 1, -1, 0),
            ("SW", -1, -1, 0), ("NT", 0, 1, 1), ("NB", 0, 1, -1), ("ST", 0, -1, 1), ("SB", 0, -1, -1),
            ("ET", 1, 0, 1), ("EB", 1, 0, -1), ("WT", -1, 0, 1), ("WB", -1, 0, -1)]
LBM_FLUID, LBM_OBSTACLE, LBM_ACCEL = 0, 1, 2


def lbm_inputs(nx: int, ny: int, nz: int, seed: int, variant: str = "cavity"):
    """Lid-driven-cavity-like grid: OBSTACLE on all 6 faces, ACCEL on the interior layer
    z = nz-2, fluid elsewhere.  f [19][nz][ny][nx] fp32 SoA.  Fluid f_i = w_i(1+1e-3 U[-1,1)),
    obstacle f_i = w_i.  variant 'rest': all fluid interior, f_i = w_i exactly, no ACCEL."""
    g = rng(seed)
    w = np.array([1 / 3] + [1 / 18] * 6 + [1 / 36] * 12, np.float64)
    flags = np.zeros((nz, ny, nx), np.uint32)
    flags[0, :, :] = flags[-1, :, :] = LBM_OBSTACLE
    flags[:, 0, :] = flags[:, -1, :] = LBM_OBSTACLE
    flags[:, :, 0] = flags[:, :, -1] = LBM_OBSTACLE
    f = np.empty((19, nz, ny, nx), np.float32)
    if variant == "rest":
        for i in range(19):
            f[i] = np.float32(w[i])
        return f, flags
    if nz >= 4:
        flags[nz - 2, 1:-1, 1:-1] = LBM_ACCEL
    for i in range(19):
        f[i] = (w[i] * (1.0 + 1e-3 * g.uniform(-1, 1, size=(nz, ny, nx)))).astype(np.float32)
        f[i][flags == LBM_OBSTACLE] = np.float32(w[i])
    return f, flags


def spmv_inputs(R: int, seed: int, mean_len: int = 32, variant: str = "random"):
    """R x R sparse matrix in CSR with sorted columns; row length min(R, Geometric(1/mean_len));
    values U[0,1); x U[0,1).  variants: 'identity', 'perm' (permutation matrix), 'int'."""
    g = rng(seed)
    if variant in ("identity", "perm"):
        cols = np.arange(R, dtype=np.int32) if variant == "identity" else g.permutation(R).astype(np.int32)
        row_ptr = np.arange(R + 1, dtype=np.int32)
        vals = np.ones(R, np.float32)
        x = g.uniform(0, 1, size=R).astype(np.float32)
        return row_ptr, cols, vals, x
    lens = np.minimum(g.geometric(1.0 / mean_len, size=R), R).astype(np.int64)
    row_ptr = np.zeros(R + 1, np.int64)
    np.cumsum(lens, out=row_ptr[1:])
    nnz = int(row_ptr[-1])
    cols = np.empty(nnz, np.int32)
    for r in range(R):
        l = int(lens[r])
        if l * 4 > R:
            c = g.choice(R, size=l, replace=False)
        else:
            c = np.unique(g.integers(0, R, size=2 * l + 8))
            while c.size < l:
                c = np.unique(np.concatenate([c, g.integers(0, R, size=l)]))
            c = g.permutation(c)[:l]
        cols[row_ptr[r]:row_ptr[r + 1]] = np.sort(c)
    if variant == "int":
        vals = g.integers(1, 4, size=nnz).astype(np.float32)
        x = g.integers(0, 4, size=R).astype(np.float32)
    else:
        vals = g.uniform(0, 1, size=nnz).astype(np.float32)
        x = g.uniform(0, 1, size=R).astype(np.float32)
    return row_ptr.astype(np.int32), cols, vals, x


def histo_inputs(N: int, nbins: int, seed: int, variant: str = "skewed"):
    """u32 bin indices in [0,nbins).  'skewed': clamp(round(Normal(nbins/2, nbins/32)));
    'uniform'; 'constant' (all = nbins/3); 'each' (every bin exactly N//nbins times, shuffled)."""
    g = rng(seed)
    if variant == "skewed":
        v = np.clip(np.rint(g.normal(nbins / 2, nbins / 32, size=N)), 0, nbins - 1)
    elif variant == "uniform":
        v = g.integers(0, nbins, size=N)
    elif variant == "constant":
        v = np.full(N, nbins // 3)
    elif variant == "each":
        v = g.permutation(np.repeat(np.arange(nbins), N // nbins))
    else:
        raise ValueError(variant)
    return v.astype(np.uint32)


def bfs_inputs(V: int, seed: int, variant: str = "random"):
    """Undirected graph as CSR (row_ptr int32 [V+1], col int32, neighbour lists sorted).
    'random': each node draws U{1..11} uniform neighbours (mean 6), symmetrised, deduped, no
    self loops.  'path', 'star', 'two' (two disconnected paths)."""
    g = rng(seed)
    if variant == "random":
        deg = g.integers(1, 12, size=V)
        src = np.repeat(np.arange(V), deg)
        dst = g.integers(0, V, size=src.size)
    elif variant == "path":
        src, dst = np.arange(V - 1), np.arange(1, V)
    elif variant == "star":
        src, dst = np.zeros(V - 1, np.int64), np.arange(1, V)
    elif variant == "two":
        h = V // 2
        src = np.concatenate([np.arange(h - 1), np.arange(h, V - 1)])
        dst = src + 1
    else:
        raise ValueError(variant)
    keep = src != dst
    s = np.concatenate([src[keep], dst[keep]])
    d = np.concatenate([dst[keep], src[keep]])
    key = np.unique(s.astype(np.int64) * V + d)
    s, d = key // V, key % V
    row_ptr = np.zeros(V + 1, np.int64)
    np.add.at(row_ptr, s + 1, 1)
    row_ptr = np.cumsum(row_ptr)
    return row_ptr.astype(np.int32), d.astype(np.int32)


# --------------------------------------------------------------------------- NEXT-3 fft
def fft_inputs(batch: int, n: int, seed: int, variant: str = "uniform"):
    """Complex fp32 signals [batch, n, 2] (re, im interleaved), Parboil-fft-like batches of 1-D
    transforms.  'uniform': re, im ~ U[-1,1); 'impulse': x[b, b % n] = 1; 'tone': x[b, j] =
    exp(2 pi i m j / n) with m = b % n (rounded to fp32)."""
    g = rng(seed)
    if variant == "uniform":
        x = g.uniform(-1, 1, size=(batch, n, 2))
    elif variant == "impulse":
        x = np.zeros((batch, n, 2))
        x[np.arange(batch), np.arange(batch) % n, 0] = 1.0
    elif variant == "tone":
        m = (np.arange(batch) % n)[:, None]
        ph = 2 * np.pi * np.mod(m * np.arange(n)[None, :], n) / n
        x = np.stack([np.cos(ph), np.sin(ph)], axis=-1)
    else:
        raise ValueError(variant)
    return np.ascontiguousarray(x.astype(np.float32))


# --------------------------------------------------------------------------- NEXT-3 tpacf
def tpacf_edges(bins_per_dec: int = 5, min_arcmin: float = 1.0, max_arcmin: float = 10000.0):
    """Parboil tpacf's bin boundaries as fp32 cosines, strictly decreasing: the angles
    10^(log10(min) + k / bins_per_dec) arcmin, k = 0 .. decades * bins_per_dec (21 edges ->
    22 counters with the two open ends)."""
    nb = int(round(math.log10(max_arcmin / min_arcmin) * bins_per_dec))
    ang = 10.0 ** (math.log10(min_arcmin) + np.arange(nb + 1) / bins_per_dec) / 60.0 * math.pi / 180.0
    e = np.cos(ang).astype(np.float32)
    assert np.all(np.diff(e) < 0)
    return e


def tpacf_inputs(n: int, seed: int, variant: str = "clustered"):
    """Unit vectors float32 [n, 3] (a sky catalogue as Cartesian points, Parboil tpacf's input
    after its ra/dec conversion).  'clustered': 60 % of the points in 64 Gaussian clumps of
    0.5-5 degrees on the sphere, 40 % uniform (galaxy-catalogue-like: every angular scale of the
    bins is populated); 'uniform'.  Normalised in fp64, then rounded to fp32."""
    g = rng(seed)
    def sphere(m):
        v = g.normal(size=(m, 3))
        return v / np.linalg.norm(v, axis=1, keepdims=True)
    if variant == "uniform":
        p = sphere(n)
    elif variant == "clustered":
        nc = int(0.6 * n)
        centres = sphere(64)
        which = g.integers(0, 64, size=nc)
        sig = g.uniform(0.5, 5.0, size=64)[which] * math.pi / 180.0
        p = np.concatenate([centres[which] + g.normal(size=(nc, 3)) * sig[:, None], sphere(n - nc)])
        p = p[g.permutation(n)]
        p /= np.linalg.norm(p, axis=1, keepdims=True)
    else:
        raise ValueError(variant)
    return np.ascontiguousarray(p.astype(np.float32))
