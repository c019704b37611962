"""Pins for the shared seeded generator (inputs/gen.c): SURVEY.md §8(d) "Generator"."""
import numpy as np

import inputs

M64 = (1 << 64) - 1


def py_mix(z):
    z &= M64
    z ^= z >> 30; z = (z * 0xBF58476D1CE4E5B9) & M64
    z ^= z >> 27; z = (z * 0x94D049BB133111EB) & M64
    z ^= z >> 31
    return z


def py_u(seed, idx):
    return (py_mix((seed * 0x9E3779B97F4A7C15 + idx) & M64) >> 11) * 2.0 ** -53


def test_splitmix_known_value():
    # splitmix64 finaliser of 0 is 0; published first output of splitmix64(seed=0) is
    # mix(0x9E3779B97F4A7C15) = 0xE220A8397B1DCDAF (Vigna's reference sequence).
    assert inputs.mix(0) == 0
    assert inputs.mix(0x9E3779B97F4A7C15) == 0xE220A8397B1DCDAF
    for z in (1, 12345, 2**63 + 7):
        assert inputs.mix(z) == py_mix(z)


def test_uniform_matches_formula_and_is_ld_independent():
    m, n = 7, 5
    a = inputs.uniform(3, m, n)
    b = inputs.uniform(3, m, n, ld=m + 4)
    assert np.array_equal(a[:m], b[:m])
    assert np.all(b[m:] == 0)
    for (i, j) in [(0, 0), (6, 4), (3, 2)]:
        assert a[i, j] == 2.0 * py_u(3, i + j * m) - 1.0
    assert a.min() >= -1.0 and a.max() < 1.0


def test_integers_range_and_formula():
    m, n = 40, 30
    a = inputs.integers(1, m, n)
    assert a.min() >= -8 and a.max() <= 8 and np.all(a == np.floor(a))
    assert a[5, 7] == np.floor(17 * py_u(1, 5 + 7 * m)) - 8
    assert len(np.unique(a)) == 17


def test_tri_dd_structure():
    n = 16
    L = inputs.tri_dd(4, n, lower=True, fill=np.nan)
    assert np.all(np.isnan(L[np.triu_indices(n, 1)]))
    d = np.diag(L)
    assert np.all((d >= 1) & (d < 2))
    off = L[np.tril_indices(n, -1)]
    assert np.all(np.abs(off) <= 1.0 / (2 * n))


def test_fills_do_not_depend_on_thread_count():
    """Counter-based: the same matrices at any OpenMP thread count (bench.py's rank 0 raises
    it above torchrun's OMP_NUM_THREADS=1)."""
    import numpy as np
    outs = []
    for n in (1, 3, 8):
        inputs.set_threads(n)
        outs.append((inputs.uniform(7, 123, 77), inputs.integers(8, 50, 61), inputs.tri_dd(9, 90)))
    inputs.set_threads(1)
    for a, b in zip(outs, outs[1:]):
        assert all(np.array_equal(x, y) for x, y in zip(a, b))
