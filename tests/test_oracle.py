"""Pins for the CPU oracle (oracle/) -- each checks it against something other than itself:
values worked by hand (tests/golden/), closed forms, invariants, a textbook routine, and
exact rational arithmetic.  CPU only.

Readings referenced: G1 update formula/op order, G2 boundary conditions,
G5/G6 initial field and boundary data, G7 norm.
"""
import math
from fractions import Fraction

import numpy as np
import pytest

import oracle
from inputs import gen


# ---------------------------------------------------------------------------------- helpers
def _read_golden(path):
    rows = {}
    with open(path) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            key, *vals = line.split()
            rows.setdefault(key, []).append(vals)
    return rows


def _f(vals):
    return [float(v) for v in vals]


# ---------------------------------------------------------------------------------- golden
def test_hand_4x4(golden_dir):
    """SURVEY §8(c) hand-worked example; P:410 5-point star."""
    g = _read_golden(f"{golden_dir}/hand4x4.txt")
    init = np.array([_f(r) for r in g["init"]], dtype=np.float32)
    for k in (1, 2, 3):
        out, sums = oracle.jacobi_run(init, k, "dirichlet", norm_every=1)
        want = np.array([_f(r) for r in g[f"iter{k}"]], dtype=np.float32)
        assert np.array_equal(out[1:3, 1:3], want)
        assert sums[k - 1] == float(g[f"sumsq{k}"][0][0])
        # fixed data never changes (invariant 2)
        assert np.array_equal(out[0], init[0]) and np.array_equal(out[3], init[3])
        assert np.array_equal(out[:, 0], init[:, 0]) and np.array_equal(out[:, 3], init[:, 3])
    fixed = np.array([_f(r) for r in g["fixed"]], dtype=np.float32)
    out, sums = oracle.jacobi_run(init, 40, "dirichlet", norm_every=1)
    assert np.array_equal(out[1:3, 1:3], fixed)
    assert sums[-1] == 0.0


def test_hand_4x4_exact_rationals(golden_dir):
    """Independent brute force in exact rationals: the fixed point solves the 4 linear
    equations u = (l+r+t+b)/4 exactly (Cramer by Fraction Gaussian elimination)."""
    g = _read_golden(f"{golden_dir}/hand4x4.txt")
    init = [[Fraction(v) for v in r] for r in g["init"]]
    # unknowns a=u11 b=u12 c=u21 d=u22 ; 4u - neighbours = boundary
    A = [[4, -1, -1, 0], [-1, 4, 0, -1], [-1, 0, 4, -1], [0, -1, -1, 4]]
    rhs = [init[1][0] + init[0][1], init[1][3] + init[0][2],
           init[2][0] + init[3][1], init[2][3] + init[3][2]]
    M = [[Fraction(x) for x in row] + [rhs[i]] for i, row in enumerate(A)]
    for c in range(4):
        p = next(r for r in range(c, 4) if M[r][c] != 0)
        M[c], M[p] = M[p], M[c]
        for r in range(4):
            if r != c and M[r][c] != 0:
                f = M[r][c] / M[c][c]
                M[r] = [x - f * y for x, y in zip(M[r], M[c])]
    sol = [M[i][4] / M[i][i] for i in range(4)]
    out, _ = oracle.jacobi_run(np.array([[float(v) for v in r] for r in init], np.float32), 60, "dirichlet")
    assert [Fraction(float(v)) for v in out[1:3, 1:3].ravel()] == sol


def test_ring_two_rows(golden_dir):
    """Periodic 2-row example (reading G2, Listing 1)."""
    g = _read_golden(f"{golden_dir}/ring2row.txt")
    rows = np.array([_f(r) for r in g["init"]], dtype=np.float32)
    init = np.vstack([rows[1], rows[0], rows[1], rows[0]])  # halo rows = wrap
    for k in (1, 2):
        out, sums = oracle.jacobi_run(init, k, "ring", norm_every=1)
        want = np.array([_f(r) for r in g[f"iter{k}"]], dtype=np.float32)
        assert np.array_equal(out[1:3], want)
        assert sums[k - 1] == float(g[f"sumsq{k}"][0][0])
        # the returned halo rows hold the wrapped rows
        assert np.array_equal(out[0], out[2]) and np.array_equal(out[3], out[1])
    # limit: linear ramp 4 + 4x/3 (closed form of the ring problem with constant columns)
    out, _ = oracle.jacobi_run(init, 400, "ring")
    ramp = 4 + 4 * np.arange(4) / 3
    assert np.allclose(out[1:3], ramp[None, :], atol=2e-6)


def test_association_cases(golden_dir):
    """Reading G1 operation order + round-to-nearest-even + no FTZ, on single-point grids."""
    g = _read_golden(f"{golden_dir}/association.txt")
    for case, vals in g.items():
        l, r, t, b, want = [float.fromhex(v) for v in vals[0]]
        a = np.zeros((3, 3), np.float32)
        a[1, 0], a[1, 2], a[0, 1], a[2, 1] = l, r, t, b
        out, _ = oracle.jacobi_run(a, 1, "dirichlet")
        assert out[1, 1] == np.float32(want), case


# ---------------------------------------------------------------------------------- generator
def test_splitmix64_known_vectors():
    """Published splitmix64 outputs for state 0 (Vigna's reference; first three outputs)."""
    golden = np.uint64(0x9E3779B97F4A7C15)
    with np.errstate(over="ignore"):
        states = np.array([0, 1, 2], np.uint64) * golden  # mixer input before the +golden step
    out = gen.splitmix64(states)
    assert [int(v) for v in out] == [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F]


def test_generator_layout():
    nx, ny = 16, 8
    g = gen.global_field(nx, ny, "ring", seed=7)
    assert g.dtype == np.float32 and g.shape == (ny + 2, nx)
    assert np.array_equal(g[0], g[ny]) and np.array_equal(g[ny + 1], g[1])
    interior = g[1:ny + 1, 1:nx - 1]
    assert interior.min() >= 0 and interior.max() < 1
    assert np.all(interior * 2 ** 24 == np.floor(interior * 2 ** 24))  # 24-bit values
    assert g[1 + ny // 4, 0] == np.float32(1.0)  # sin(pi/2)
    d = gen.global_field(nx, ny, "dirichlet", seed=7)
    assert np.array_equal(d[1:ny + 1, 1:nx - 1], interior)
    assert d[0, nx // 2] == np.float32(math.sin(math.pi * (nx // 2) / (nx - 1)))
    assert not d[ny + 1].any() and not d[1:ny + 1, 0].any() and not d[1:ny + 1, nx - 1].any()
    for topo in ("ring", "dirichlet"):
        full = gen.global_field(nx, ny, topo, seed=3)
        for P in (1, 2, 4, 8):
            for r in range(P):
                assert np.array_equal(gen.rank_slab(full, r, P), gen.slab_field(nx, ny, r, P, topo, seed=3))


# ---------------------------------------------------------------------------------- invariants
@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
def test_constant_field_is_fixed(topology):
    a = np.full((10, 12), 0.3, np.float32)
    out, sums = oracle.jacobi_run(a, 7, topology, norm_every=1)
    assert np.array_equal(out, a) and not sums.any()


def test_dirichlet_cells_never_change():
    g = gen.global_field(20, 12, "dirichlet", seed=11)
    out, _ = oracle.jacobi_run(g, 13, "dirichlet")
    for sl in (np.s_[0, :], np.s_[-1, :], np.s_[:, 0], np.s_[:, -1]):
        assert np.array_equal(out[sl].view(np.uint32), g[sl].view(np.uint32))


@pytest.mark.parametrize("topology", ["ring", "dirichlet"])
def test_mirror_symmetry(topology):
    """IEEE + is commutative, so x-mirrored data gives an x-mirrored result bitwise."""
    g = gen.global_field(17, 10, topology, seed=5)
    g[:, 9:] = g[:, :8][:, ::-1]  # make columns i and NX-1-i equal
    out, _ = oracle.jacobi_run(g, 9, topology)
    assert np.array_equal(out, out[:, ::-1])
    if topology == "dirichlet":  # y-mirror too
        h = g.copy()
        h[6:] = h[:6][::-1]
        out, _ = oracle.jacobi_run(h, 9, topology)
        assert np.array_equal(out, out[::-1])


def test_max_principle_and_power_of_two_scaling():
    g = gen.global_field(24, 16, "dirichlet", seed=9)
    out, _ = oracle.jacobi_run(g, 30, "dirichlet")
    assert out.min() >= g.min() and out.max() <= g.max()
    out8, _ = oracle.jacobi_run(g * np.float32(8), 30, "dirichlet")
    assert np.array_equal(out8, out * np.float32(8))
    outq, _ = oracle.jacobi_run(g * np.float32(2 ** -20), 30, "dirichlet")
    assert np.array_equal(outq, out * np.float32(2 ** -20))


def test_subnormal_front_no_ftz():
    """Zero field, unit left column, uniform rows (ring): the front at column k after k
    iterations is exactly 4^-k (only the left neighbour is non-zero), including subnormals
    2^-128 .. 2^-148 which FTZ/DAZ would flush."""
    nx, ny = 90, 2
    a = np.zeros((ny + 2, nx), np.float32)
    a[:, 0] = 1.0
    for k in (1, 10, 63, 64, 70, 74):
        out, _ = oracle.jacobi_run(a, k, "ring")
        assert out[1, k] == np.float32(2.0 ** (-2 * k)), k
        assert out[1, k + 1] == 0.0
    out, _ = oracle.jacobi_run(a, 75, "ring")
    assert out[1, 75] == 0.0  # 2^-150: tie, rounds to even (zero)
    assert out[1, 74] > 0


# ---------------------------------------------------------------------------------- closed forms
@pytest.mark.parametrize("nx,ny,iters,tol", [(8, 6, 600, 2e-7), (16, 14, 3000, 1e-6)])
def test_dirichlet_sin_sinh_discrete_harmonic(nx, ny, iters, tol):
    """Fixed point = discrete harmonic function u[j][i] = sin(pi i/(NX-1)) sinh(lam (NY+1-j))
    / sinh(lam (NY+1)), cosh(lam) = 2 - cos(pi/(NX-1)) (separation of variables)."""
    g = gen.global_field(nx, ny, "dirichlet", zero_init=True)
    out, _ = oracle.jacobi_run(g, iters, "dirichlet")
    lam = math.acosh(2 - math.cos(math.pi / (nx - 1)))
    j = np.arange(ny + 2)[:, None]
    i = np.arange(nx)[None, :]
    exact = np.sin(np.pi * i / (nx - 1)) * np.sinh(lam * (ny + 1 - j)) / math.sinh(lam * (ny + 1))
    err = np.abs(out[1:ny + 1, 1:nx - 1] - exact[1:ny + 1, 1:nx - 1]).max()
    assert err < tol


def test_continuous_limit_is_second_order():
    """Against sin(pi x) sinh(pi y)/sinh(pi) the discretisation error falls ~4x per halving."""
    errs = []
    for m in (8, 16):
        nx, ny = m + 1, m - 1  # h = 1/m in both directions
        g = gen.global_field(nx, ny, "dirichlet", zero_init=True)
        g[0] = np.sin(np.pi * np.arange(nx) / m).astype(np.float32)
        out, _ = oracle.jacobi_run(g, 4000, "dirichlet")
        x = np.arange(nx) / m
        y = 1 - np.arange(ny + 2) / m  # row 0 is y = 1
        ex = np.sin(np.pi * x)[None, :] * np.sinh(np.pi * y)[:, None] / math.sinh(math.pi)
        errs.append(np.abs(out - ex)[1:ny + 1, 1:nx - 1].max())
    assert 3.0 < errs[0] / errs[1] < 5.0


def test_ring_closed_form():
    """u = sin(2 pi gy/NY) sinh(mu (NX-1-i))/sinh(mu (NX-1)), cosh mu = 2 - cos(2 pi/NY)."""
    nx, ny = 16, 16
    g = gen.global_field(nx, ny, "ring", zero_init=True)
    out, _ = oracle.jacobi_run(g, 3000, "ring")
    mu = math.acosh(2 - math.cos(2 * math.pi / ny))
    gy = np.arange(ny)[:, None]
    i = np.arange(nx)[None, :]
    ex = np.sin(2 * np.pi * gy / ny) * np.sinh(mu * (nx - 1 - i)) / math.sinh(mu * (nx - 1))
    assert np.abs(out[1:ny + 1] - ex).max() < 1e-6


def test_norm_decay_rate_is_jacobi_spectral_radius():
    """||d_{k+2}|| / ||d_k|| -> rho^2, rho = (cos(pi/(NX-1)) + cos(pi/(NY+1)))/2 (Jacobi
    iteration matrix of the 5-point Laplacian)."""
    nx, ny = 18, 16
    g = gen.global_field(nx, ny, "dirichlet", seed=1)
    _, sums = oracle.jacobi_run(g, 302, "dirichlet", norm_every=1)
    rho = (math.cos(math.pi / (nx - 1)) + math.cos(math.pi / (ny + 1))) / 2
    ratio = math.sqrt(sums[300] / sums[298])
    assert abs(ratio - rho ** 2) < 1e-4


def test_dense_matrix_jacobi_textbook():
    """Textbook x <- D^-1 (b - (L+U) x) on the assembled 5-point matrix, float64."""
    nx, ny = 8, 6
    g = gen.global_field(nx, ny, "dirichlet", seed=3)
    nxi = nx - 2
    N = ny * nxi
    A = np.zeros((N, N))
    b = np.zeros(N)
    idx = lambda j, i: (j - 1) * nxi + (i - 1)
    for j in range(1, ny + 1):
        for i in range(1, nx - 1):
            p = idx(j, i)
            A[p, p] = 4.0
            for jj, ii in ((j, i - 1), (j, i + 1), (j - 1, i), (j + 1, i)):
                if 1 <= jj <= ny and 1 <= ii <= nx - 2:
                    A[p, idx(jj, ii)] = -1.0
                else:
                    b[p] += float(g[jj, ii])
    D = np.diag(A)
    R = A - np.diag(D)
    x = np.array([float(g[j, i]) for j in range(1, ny + 1) for i in range(1, nx - 1)])
    for _ in range(50):
        x = (b - R @ x) / D
    out, _ = oracle.jacobi_run(g, 50, "dirichlet")
    assert np.abs(out[1:ny + 1, 1:nx - 1].ravel() - x).max() < 2e-6


def test_windowed_oracle_equals_global_oracle():
    """The sampling method of tests/test_gpu_fullsize.py: k iterations of the oracle on a window
    of rows [y0-k-1, y1+k+1] with fixed edge rows reproduce rows y0..y1 of the global run
    (dependency cone of k rows), including windows across the ring wrap-around."""
    import sys, os
    sys.path.insert(0, os.path.dirname(__file__))
    nx, ny, k = 40, 30, 4
    full, _ = oracle.jacobi_run(gen.global_field(nx, ny, "ring"), k, "ring")
    for y0, y1 in ((5, 9), (-1, 3), (26, 30), (0, 0)):
        gys = list(range(y0 - k - 1, y1 + k + 2))
        w, _ = oracle.jacobi_run(gen.rows_field(nx, ny, gys, "ring"), k, "dirichlet")
        got = w[k + 1:k + 1 + (y1 - y0 + 1)]
        want = np.array([full[1 + (gy % ny)] for gy in range(y0, y1 + 1)])
        assert np.array_equal(got, want), (y0, y1)
    # a fixed edge row only k-1 rows away does corrupt the sample: the cone really is k rows
    gys = list(range(5 - k + 1, 9 + k))
    w, _ = oracle.jacobi_run(gen.rows_field(nx, ny, gys, "ring"), k, "dirichlet")
    assert not np.array_equal(w[k - 1:k + 4], np.array([full[1 + gy] for gy in range(5, 10)]))


def test_norm_matches_consecutive_iterates():
    """The norm record equals sum((A_{k+1}-A_k)^2) recomputed from the oracle's own grids
    (d in fp32, squares summed in double) -- north_star norm, reading G7."""
    g = gen.global_field(33, 20, "ring", seed=2)
    _, sums = oracle.jacobi_run(g, 12, "ring", norm_every=5)
    assert len(sums) == 3
    for m, k in enumerate((0, 5, 10)):
        a, _ = oracle.jacobi_run(g, k, "ring")
        b, _ = oracle.jacobi_run(g, k + 1, "ring")
        d = (b[1:-1, 1:-1] - a[1:-1, 1:-1]).astype(np.float64)
        assert math.isclose(sums[m], float((d * d).sum()), rel_tol=1e-12)
