"""Pins of the CPU oracle (oracle/) to things other than itself.

Each test names the pin of DESIGN.md §4 it implements and
the passage or reading it follows. None of these tests needs a GPU.
"""
import math
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle as O

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _read_golden(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line)
    return rows


# ---------------------------------------------------------------- generator (S7)

def test_splitmix64_published_vector():
    """SplitMix64 stream for seed 1234567 equals the published reference outputs."""
    rows = _read_golden("splitmix64_seed1234567.txt")
    assert rows[0] == "seed 1234567"
    want = [int(r) for r in rows[1:]]
    got = [O.splitmix64_at(1234567, i) for i in range(len(want))]
    assert got == want


def test_rest_lattice_centred_and_mirror_exact():
    """Reading S7/item 1: centred lattice; mirror images are exact negations."""
    for n in [(5, 6, 7), (4, 4, 9)]:
        p = O.Params(n=n, spacing=0.75)
        for i in range(n[0]):
            a = O.rest_position(p, i, 1, 2)
            b = O.rest_position(p, n[0] - 1 - i, 1, 2)
            assert a[0] == -b[0] and a[1] == b[1] and a[2] == b[2]
            assert a[0] == (i - (n[0] - 1) / 2) * 0.75


def test_init_faces_velocities_and_displacements():
    p = O.Params(n=(7, 6, 9), amplitude=0.05, seed=3)
    s = O.init(p)
    n0, n1, n2 = p.n
    interior = np.zeros(p.n, bool)
    interior[1:-1, 1:-1, 1:-1] = True
    x0 = np.stack(np.meshgrid(*[(np.arange(m) - (m - 1) / 2) * p.spacing for m in p.n], indexing="ij"))
    X = s.X
    # fixed faces exactly at the rest lattice; V = 0 everywhere
    assert np.array_equal(X[:, ~interior], x0[:, ~interior])
    assert not s.V.any()
    # interior displacement in [-a, a): every component drawn
    d = (X - x0)[:, interior]
    assert np.all(np.abs(d) <= p.amplitude) and np.all(d != 0)
    # sampled nodes: counter 3g+c of the pinned generator, u = (r >> 11) * 2^-53
    for (i, j, k) in [(1, 1, 1), (3, 2, 5), (5, 4, 7)]:
        g = (i * n1 + j) * n2 + k
        for c in range(3):
            u = (O.splitmix64_at(p.seed, 3 * g + c) >> 11) / 2.0 ** 53
            assert X[c, i, j, k] == x0[c, i, j, k] + p.amplitude * (2 * u - 1)


def test_init_displacement_uniform_moments():
    p = O.Params(n=(24, 24, 24), amplitude=0.05, seed=42)
    s = O.init(p)
    x0 = np.stack(np.meshgrid(*[(np.arange(m) - (m - 1) / 2) for m in p.n], indexing="ij"))
    d = (s.X - x0)[:, 1:-1, 1:-1, 1:-1].ravel() / p.amplitude
    n = d.size
    assert abs(d.mean()) < 5 / math.sqrt(3 * n)          # U(-1,1): var 1/3
    assert abs(d.var() - 1 / 3) < 5 * math.sqrt(4 / 45 / n)
    # components independent: correlation of x and y displacements ~ 0
    dd = (s.X - x0)[:, 1:-1, 1:-1, 1:-1].reshape(3, -1)
    assert abs(np.corrcoef(dd[0], dd[1])[0, 1]) < 5 / math.sqrt(dd.shape[1])


def test_init_window_is_a_slice_of_the_full_init():
    p = O.Params(n=(9, 11, 13), seed=5)
    full = O.init(p)
    for lo, w in [((0, 0, 0), (9, 11, 13)), ((2, 3, 4), (5, 6, 7)), ((8, 10, 12), (1, 1, 1))]:
        s = O.init_window(p, lo, w)
        sl = tuple(slice(a, a + b) for a, b in zip(lo, w))
        assert np.array_equal(s.X, full.X[(slice(None),) + sl]) and not s.V.any()
    with pytest.raises(ValueError):
        O.init_window(p, (5, 0, 0), (5, 1, 1))


def test_light_cone_window_reproduces_a_full_run_node():
    """A node after S steps depends only on the initial state within distance S:
    running the oracle on a window reaching S+1 beyond it reproduces the full
    run there, bit for bit (the basis of the full-size GPU spot checks)."""
    p = O.Params(n=(20, 21, 22), seed=6)
    S = 4
    full, _ = O.run(O.init(p), S)
    for c in [(10, 10, 10), (1, 1, 1), (18, 5, 20), (6, 19, 2)]:
        lo = [max(0, c[d] - S - 1) for d in range(3)]
        hi = [min(p.n[d], c[d] + S + 2) for d in range(3)]
        win = O.init_window(p, lo, [hi[d] - lo[d] for d in range(3)])
        win, _ = O.run(win, S)
        rel = tuple(c[d] - lo[d] for d in range(3))
        assert np.array_equal(win.X[(slice(None),) + rel], full.X[(slice(None),) + tuple(c)])
        assert np.array_equal(win.V[(slice(None),) + rel], full.V[(slice(None),) + tuple(c)])


def test_init_rejects_invalid():
    for bad in [O.Params(n=(2, 5, 5)), O.Params(mass=0.0), O.Params(dt=-1.0), O.Params(k_spring=float("nan"))]:
        with pytest.raises(ValueError):
            O.init(bad)


# ---------------------------------------------------------------- spring law (S1)

def test_spring_closed_forms():
    K, L = 10.0, 1.0
    # stretched to 2L along x: f = K(2L-L)/(2L) -> g = f*(2L,0,0) = (K L, 0, 0)
    assert O.spring((0, 0, 0), (2, 0, 0), K, L) == (10.0, 0.0, 0.0)
    # compressed to L/2 along -z: pushes p away from q (g points along -d)
    g = O.spring((0, 0, 0), (0, 0, -0.5), K, L)
    assert g == (0.0, 0.0, 5.0)
    # at rest length: exactly zero
    assert O.spring((0.25, 0.5, 1.0), (1.25, 0.5, 1.0), K, L) == (0.0, 0.0, 0.0)
    # 3-4-5 triangle: d = 5, f = K*4/5 = 8, g = 8 * (3, 4, 0)
    assert O.spring((0, 0, 0), (3, 4, 0), K, L) == (24.0, 32.0, 0.0)


def test_spring_antisymmetric_bitwise():
    rng = np.random.default_rng(7)
    for _ in range(200):
        a, b = rng.normal(size=3), rng.normal(size=3)
        gab = O.spring(a, b, 3.7, 0.9)
        gba = O.spring(b, a, 3.7, 0.9)
        assert gab == tuple(-v for v in gba)


# ---------------------------------------------------------------- integrator (S4) C2, C3

def _two_mass(K, M, L, h, r0, nsteps):
    xp, xq = [-(L + r0) / 2, 0.0, 0.0], [(L + r0) / 2, 0.0, 0.0]
    vp, vq = [0.0] * 3, [0.0] * 3
    rs, ws = [r0], [0.0]
    sym = True
    for _ in range(nsteps):
        gp = O.spring(xp, xq, K, L)      # force on p
        gq = O.spring(xq, xp, K, L)      # force on q
        for c in range(3):
            vp[c] = O.velocity_1(vp[c], O.acceleration_1(gp[c], M), h)
            vq[c] = O.velocity_1(vq[c], O.acceleration_1(gq[c], M), h)
            xp[c] = O.position_1(xp[c], vp[c], h)
            xq[c] = O.position_1(xq[c], vq[c], h)
        sym = sym and xp[0] == -xq[0] and vp[0] == -vq[0]
        rs.append((xq[0] - xp[0]) - L)
        ws.append(vq[0] - vp[0])
    return np.array(rs), np.array(ws), sym


# (K, M, L): the survey's defaults, a heavy node (M != 1: a = F/M)
# and a soft spring with another rest length -- the relative coordinate's
# frequency w^2 = 2K/M must follow both K and M
TWO_MASS_CASES = [(10.0, 1.0, 1.0), (10.0, 2.5, 1.0), (3.0, 0.7, 0.8)]


@pytest.mark.parametrize("K,M,L", TWO_MASS_CASES)
def test_two_mass_oscillator_exact_discrete_solution(K, M, L):
    """C2: relative coordinate obeys symplectic Euler with w^2 = 2K/M; exact
    discrete solution r_n = r0 cos(n th) + ((r1 - r0 cos th)/sin th) sin(n th),
    th = 2 asin(h w / 2) (PAPER.md:323-326 forces ->
    accelerations (F/M) -> velocities -> positions)."""
    h, r0, N = 1e-3, 0.1, 20000
    rs, ws, sym = _two_mass(K, M, L, h, r0, N)
    w = math.sqrt(2 * K / M)
    th = 2 * math.asin(h * w / 2)
    r1 = r0 * (1 - h * h * w * w)
    n = np.arange(N + 1)
    exact = r0 * np.cos(n * th) + ((r1 - r0 * math.cos(th)) / math.sin(th)) * np.sin(n * th)
    assert np.max(np.abs(rs - exact)) / r0 < 1e-11
    # the continuous solution agrees to O(h) in phase only
    cont = r0 * np.cos(w * h * n)
    assert np.max(np.abs(rs - cont)) / r0 < 0.1
    # C3 (part): centre of mass exactly at rest (forces are exact negatives)
    assert sym


@pytest.mark.parametrize("K,M,L", TWO_MASS_CASES)
def test_two_mass_discrete_invariant(K, M, L):
    """C3: Q = w^2 + W^2 r^2 - h W^2 r w is conserved by the symplectic-Euler map, W^2 = 2K/M."""
    h, r0, N = 1e-2, 0.2, 5000
    rs, ws, _ = _two_mass(K, M, L, h, r0, N)
    W2 = 2 * K / M
    Q = ws ** 2 + W2 * rs ** 2 - h * W2 * rs * ws
    assert np.max(np.abs(Q - Q[0])) / Q[0] < 1e-12
    # whereas the true energy oscillates at O(h)
    E = ws ** 2 + W2 * rs ** 2
    assert np.max(np.abs(E - E[0])) / E[0] > 1e-4


# ---------------------------------------------------------------- grid pins C4, C5

@pytest.mark.parametrize("n,spacing,rest_len", [((6, 5, 4), 1.0, 1.0), ((5, 5, 5), 1.0, 1.0), ((4, 7, 6), 0.5, 0.5),
                                                ((6, 5, 7), 1.0, 0.8), ((5, 6, 4), 1.25, 1.0)])
def test_rest_lattice_is_exact_equilibrium(n, spacing, rest_len):
    """C4: at the rest lattice every spring has d == spacing; the two springs of
    an axis pull with exactly opposite forces (d vectors negate exactly), so the
    force is exactly 0 -- also when the lattice is pre-stressed (L != spacing) --
    and the state is bitwise unchanged after 50 steps, centre exactly 0 (C9)."""
    p = O.Params(n=n, spacing=spacing, rest_len=rest_len, amplitude=0.0, mass=1.7)
    s0 = O.init(p)
    s, st = O.run(s0, 50)
    assert np.array_equal(s.X, s0.X)
    assert not s.V.any()
    assert st.centre == (0.0, 0.0, 0.0) and st.vmax == 0.0 and st.sums == (0, 0, 0)


def _mirror_state(p, axis, seed):
    """State whose displacement is odd along `axis` about the centre plane and
    even in the other components (reading S5's Jacobi step keeps it so)."""
    rng = np.random.default_rng(seed)
    s = O.init(O.Params(n=p.n, spacing=p.spacing, rest_len=p.rest_len, amplitude=0.0))
    s.p = p
    X = s.X
    V = np.zeros_like(X)
    d = rng.uniform(-0.05, 0.05, size=X.shape)
    dv = rng.uniform(-0.01, 0.01, size=X.shape)
    interior = np.zeros(p.n, bool)
    interior[1:-1, 1:-1, 1:-1] = True
    d[:, ~interior] = 0
    dv[:, ~interior] = 0
    flip = lambda a: np.flip(a, axis=1 + axis)
    sign = np.ones((3, 1, 1, 1))
    sign[axis] = -1
    # symmetrise: f(p) = (d(p) + sign*d(m(p)))/2 is exactly (anti)symmetric after rounding? no:
    # build explicitly: keep the lower half, mirror it onto the upper half.
    m = p.n[axis]
    for arr in (d, dv):
        lower = np.take(arr, range(m // 2), axis=1 + axis)
        mirrored = np.flip(lower, axis=1 + axis) * sign
        idx = [slice(None)] * 4
        idx[1 + axis] = slice(m - m // 2, m)
        arr[tuple(idx)] = mirrored
        if m % 2 == 1:
            idx[1 + axis] = m // 2
            arr[axis][tuple(idx[1:])] = 0.0
    X = X + d
    V = dv
    s.x, s.y, s.z = (np.ascontiguousarray(X[c]) for c in range(3))
    s.vx, s.vy, s.vz = (np.ascontiguousarray(V[c]) for c in range(3))
    # the construction is exactly mirror-symmetric
    assert np.array_equal(flip(s.X) * sign, s.X) and np.array_equal(flip(s.V) * sign, s.V)
    return s


@pytest.mark.parametrize("n", [(7, 8, 6), (8, 7, 9)])
@pytest.mark.parametrize("axis", [0, 1, 2])
def test_mirror_symmetry_bitwise(n, axis):
    """C5: a displacement odd along `axis` stays exactly odd for 100 steps. Holds
    only with the pairwise sum ((g-i+g+i)+(g-j+g+j))+(g-k+g+k) (reading S13)."""
    p = O.Params(n=n)
    s0 = _mirror_state(p, axis, seed=axis * 10 + n[0])
    s, st = O.run(s0, 100)
    sign = np.ones((3, 1, 1, 1))
    sign[axis] = -1
    flip = lambda a: np.flip(a, axis=1 + axis)
    assert not np.array_equal(s.X, s0.X)
    assert np.array_equal(flip(s.X) * sign, s.X)
    assert np.array_equal(flip(s.V) * sign, s.V)
    # C9: the mirrored coordinate's centre is exactly zero
    assert st.centre[axis] == 0.0 and st.sums[axis] == 0


# ---------------------------------------------------------------- C6 brute force

def _edge_list_forces(X, K, L):
    """Each spring evaluated once along every axis (edge list), +g on one end and
    -g on the other; fixed faces zeroed. Independent of the node-centric loop."""
    F = np.zeros_like(X)
    for a in range(3):
        lo = [slice(None)] * 4
        hi = [slice(None)] * 4
        lo[1 + a] = slice(0, -1)
        hi[1 + a] = slice(1, None)
        dvec = X[tuple(hi)] - X[tuple(lo)]
        d = np.sqrt((dvec[0] * dvec[0] + dvec[1] * dvec[1]) + dvec[2] * dvec[2])
        g = (K * (d - L)) / d * dvec
        F[tuple(lo)] += g
        F[tuple(hi)] -= g
    F[:, 0, :, :] = F[:, -1, :, :] = 0
    F[:, :, 0, :] = F[:, :, -1, :] = 0
    F[:, :, :, 0] = F[:, :, :, -1] = 0
    return F


def test_forces_match_edge_list_brute_force():
    p = O.Params(n=(9, 8, 7), amplitude=0.2, seed=2)
    s = O.init(p)
    F = np.stack(O.forces(s))
    Fb = _edge_list_forces(s.X, p.k_spring, p.rest_len)
    scale = np.max(np.abs(Fb))
    assert scale > 0.1
    assert np.max(np.abs(F - Fb)) <= 8 * np.finfo(float).eps * scale


def test_trajectory_matches_edge_list_integrator():
    """C6 over 100 steps: an independent numpy edge-list integrator agrees to ~1e-16 rel."""
    p = O.Params(n=(8, 9, 10), amplitude=0.05, seed=5)
    s0 = O.init(p)
    X, V = s0.X.copy(), s0.V.copy()
    interior = np.zeros(p.n, bool)
    interior[1:-1, 1:-1, 1:-1] = True
    for _ in range(100):
        F = _edge_list_forces(X, p.k_spring, p.rest_len)
        V = np.where(interior, V + (F / p.mass) * p.dt, V)
        X = np.where(interior, X + V * p.dt, X)
    s, _ = O.run(s0, 100)
    assert np.max(np.abs(s.X - X)) < 1e-15
    assert np.max(np.abs(s.V - V)) < 1e-15 * 50  # |V| ~ 1e-2 .. rel ~1e-14


def test_step_is_the_five_kernels_in_order():
    """forces -> accelerations -> velocities -> positions -> centers."""
    p = O.Params(n=(6, 7, 8), seed=9)
    s = O.init(p)
    s1, st = O.step(s)
    f = O.forces(s)
    a = O.accelerations(p, f)
    v = [s.vx.copy(), s.vy.copy(), s.vz.copy()]
    O.velocities(p, a, v)
    xn = O.positions(p, [s.x, s.y, s.z], v)
    assert np.array_equal(np.stack(xn), s1.X) and np.array_equal(np.stack(v), s1.V)


# ---------------------------------------------------------------- C7 energy

def _energies(s, p):
    X, V = s.X, s.V
    kin = 0.5 * p.mass * np.sum(V * V)
    pot = 0.0
    for a in range(3):
        lo = [slice(None)] * 4
        hi = [slice(None)] * 4
        lo[1 + a] = slice(0, -1)
        hi[1 + a] = slice(1, None)
        dv = X[tuple(hi)] - X[tuple(lo)]
        d = np.sqrt(np.sum(dv * dv, axis=0))
        pot += 0.5 * p.k_spring * np.sum((d - p.rest_len) ** 2)
    F = np.stack(O.forces(s))
    return kin + pot, kin + pot + 0.5 * p.dt * np.sum(F * V)


@pytest.mark.parametrize("h,steps", [(1e-3, 2000), (1e-2, 200)])
@pytest.mark.parametrize("M,L", [(1.0, 1.0), (2.5, 0.8)])
def test_energy_bounded_modified_energy_conserved(h, steps, M, L):
    """C7: E = sum(M v^2/2) + sum(K (d-L)^2/2) stays bounded; the modified energy
    E + (h/2) sum(F.v) of symplectic Euler is conserved to O(h^2) -- for any mass
    and rest length (the energy uses M and L explicitly, so a dynamics with the
    wrong mass or rest length does not conserve it)."""
    p = O.Params(n=(8, 8, 8), amplitude=0.05, seed=11, dt=h, mass=M, rest_len=L)
    s = O.init(p)
    Es, Hs = [], []
    for t in range(steps):
        E, H = _energies(s, p)
        Es.append(E)
        Hs.append(H)
        s, _ = O.step(s)
    Es, Hs = np.array(Es), np.array(Hs)
    devH = np.max(np.abs(Hs - Hs[0])) / Hs[0]
    devE = np.max(np.abs(Es - Es[0])) / Es[0]
    assert devH < 3e-7 * (h / 1e-3) ** 2
    assert devH < devE / 5
    half = steps // 2
    assert np.max(np.abs(Es[half:] - Es[0])) < 2.0 * np.max(np.abs(Es[:half] - Es[0])) + 1e-12


def test_modified_energy_scales_h_squared():
    devs = {}
    for h, steps in [(1e-3, 1000), (1e-2, 100)]:
        p = O.Params(n=(7, 7, 7), amplitude=0.05, seed=12, dt=h)
        s = O.init(p)
        Hs = []
        for _ in range(steps):
            Hs.append(_energies(s, p)[1])
            s, _ = O.step(s)
        devs[h] = np.max(np.abs(np.array(Hs) - Hs[0])) / Hs[0]
    ratio = devs[1e-2] / devs[1e-3]
    assert 30 < ratio < 300


# ---------------------------------------------------------------- C8 linear chain

# (spacing s, rest length L, mass M): the survey's defaults, a lattice under
# tension (L < s) with a heavy node, and one under tension with a light node
# and a longer lattice spacing. Pre-stress stiffens the chain laterally: the
# four fixed lateral springs of each node (j, k faces of the (n0,3,3) chain)
# pull back a longitudinal displacement u with K(1 - L/s) u each.
CHAIN_CASES = [(1.0, 1.0, 1.0), (1.0, 0.8, 2.5), (1.25, 1.0, 0.7)]


@pytest.mark.parametrize("s_,L,M", CHAIN_CASES)
@pytest.mark.parametrize("m", [1, 2, 3])
def test_small_amplitude_chain_matches_normal_mode(m, s_, L, M):
    """C8: a longitudinal mode of the (n0,3,3) chain with fixed ends follows the
    linearised closed form M u_i'' = K (u_{i+1} - 2 u_i + u_{i-1}) - 4 K (1 - L/s) u_i,
    i.e. w_m^2 = (4K/M) (sin^2(pi m / (2 (n0-1))) + 1 - L/s), under symplectic
    Euler (th = 2 asin(h w / 2)) up to O(eps^2). With L == s it is the
    linear-chain form w_m = 2 sqrt(K/M) sin(pi m / (2 (n0-1))) of SURVEY §8(c) C8."""
    n0, eps, steps = 17, 1e-4, 500
    p = O.Params(n=(n0, 3, 3), amplitude=0.0, spacing=s_, rest_len=L, mass=M)
    s = O.init(p)
    i = np.arange(n0)
    shape = eps * np.sin(np.pi * m * i / (n0 - 1))
    s.x[1:-1, 1, 1] += shape[1:-1]
    x0 = s.x.copy()
    y0, z0 = s.y.copy(), s.z.copy()
    s, _ = O.run(s, steps)
    u = s.x[:, 1, 1] - x0[:, 1, 1] + np.where((i > 0) & (i < n0 - 1), shape, 0)
    h, K = p.dt, p.k_spring
    w = math.sqrt(4 * K / M * (math.sin(math.pi * m / (2 * (n0 - 1))) ** 2 + 1 - L / s_))
    th = 2 * math.asin(h * w / 2)
    r1 = 1 - h * h * w * w
    amp = math.cos(steps * th) + ((r1 - math.cos(th)) / math.sin(th)) * math.sin(steps * th)
    exact = shape * amp
    assert np.max(np.abs(u - exact)) / eps < 1e-6
    # the mode has moved well away from its start (the check is not vacuous)
    assert np.max(np.abs(u - shape)) / eps > 1e-3
    # lateral components untouched
    assert np.array_equal(s.y, y0) and np.array_equal(s.z, z0)
    assert not s.vy.any() and not s.vz.any()


# ---------------------------------------------------------------- C9 stats

def test_centers_exact_fixed_point_sum():
    """C9: sums are exactly sum(round_half_even(x * 2^60)) (Python Fractions),
    centre agrees with math.fsum/N, vmax with numpy."""
    p = O.Params(n=(6, 5, 7), seed=4, amplitude=0.3)
    s = O.init(p)
    s, st = O.run(s, 3)
    N = s.x.size
    for c, arr in enumerate((s.x, s.y, s.z)):
        exact = sum(round(Fraction(float(v)) * 2 ** 60) for v in arr.ravel())
        assert st.sums[c] == exact
        assert abs(st.centre[c] - math.fsum(arr.ravel()) / N) <= 1e-18 + 4e-16 * abs(st.centre[c])
    v2 = ((s.vx * s.vx + s.vy * s.vy) + s.vz * s.vz).max()
    assert st.vmax == math.sqrt(v2)
    assert st.vmax2_bits == np.float64(v2).view(np.uint64)


def test_centers_tiny_values_round_half_even():
    """Quantisation below 2^-60 rounds half to even and is sign-symmetric."""
    p = O.Params(n=(3, 3, 3))
    s = O.empty(p)
    s.x.ravel()[:4] = [2.0 ** -61, -(2.0 ** -61), 3 * 2.0 ** -61, 2.0 ** -62]
    st = O.centers(s)
    assert st.sums[0] == 0 + 0 + 2 + 0


# ---------------------------------------------------------------- toy stencil

def test_stencil3_brute_force():
    a = np.random.default_rng(0).normal(size=14)
    b = O.stencil3(a)
    for i in range(1, 13):
        assert b[i] == a[i - 1] + a[i] + a[i + 1]
    assert b[0] == 0 and b[13] == 0


# ---- reduce_exact: the reduction clause's definition (S15 generalised)
def test_reduce_exact_pins():
    """Pins of oracle.reduce_exact against things that fix it independently:
    math.fsum on dyadic data the quantisation leaves exact, hand-computed
    half-even ties, numpy min/max, IEEE signed-zero order, and the C oracle's
    own "centers" sums of a Somier state."""
    import math

    rng = np.random.default_rng(4)
    a = rng.integers(-2 ** 40, 2 ** 40, 1000) * 2.0 ** -30  # 30 fractional bits: exact at scale 30
    v, S = O.reduce_exact(a, 0, 1000, "sum", 30)
    assert v == math.fsum(a) and S == sum(int(x * 2 ** 30) for x in a)
    assert O.reduce_exact([0.5, 1.5, 2.5, -0.5, -1.5], 0, 5, "sum", 0) == (0.0 + 2 + 2 - 0 - 2, 2)
    assert O.reduce_exact([0.5, 1.5, 2.5, -0.5, -1.5], 1, 3, "sum", 0)[1] == 2 + 2 - 0
    b = rng.standard_normal(333)
    assert O.reduce_exact(b, 0, 333, "min")[0] == b.min() and O.reduce_exact(b, 0, 333, "max")[0] == b.max()
    assert math.copysign(1, O.reduce_exact([0.0, -0.0, 0.0], 0, 3, "min")[0]) == -1
    assert math.copysign(1, O.reduce_exact([-0.0, 0.0, -0.0], 0, 3, "max")[0]) == 1
    assert math.isnan(O.reduce_exact([1.0, math.nan], 0, 2, "max")[0])
    assert O.reduce_exact([], 0, 0, "min")[0] == math.inf
    with pytest.raises(ValueError):
        O.reduce_exact([2.0 ** 34], 0, 1, "sum", 60)
    # the Somier centre sums of the C oracle are this reduction of the positions at scale 60
    p = O.Params(n=(7, 6, 9), seed=3)
    s, st = O.run(O.init(p), 2)
    for c in range(3):
        assert O.reduce_exact(s.X[c].ravel(), 0, s.X[c].size, "sum", 60)[1] == st.sums[c]
