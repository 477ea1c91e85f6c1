"""The layer index's colouring (spade_layer_assign, host-only; layers of
mutually non-intersecting polygons).  Pinned to what fixes it independently of the code: every
conflict pair lands in different layers (validity), the greedy bound layers <= max degree + 1,
closed forms (no conflicts -> one layer; the complete graph K_n -> n layers; a bipartite graph K_m,n
-> 2 layers, an odd cycle -> 3), and argument checks.  No GPU needed."""
import numpy as np
import pytest

import paper_conf_icde_doraiswamyf22_b200 as sp


def _valid(a, b, lay):
    a, b = np.asarray(a), np.asarray(b)
    ne = a != b
    return bool(np.all(lay[a[ne]] != lay[b[ne]]))


def test_closed_forms():
    lay, L = sp.layer_assign([], [], 7)
    assert L == 1 and np.all(lay == 0)
    n = 6
    a, b = np.triu_indices(n, 1)
    lay, L = sp.layer_assign(a, b, n)
    assert L == n and sorted(lay.tolist()) == list(range(n))
    a = np.repeat(np.arange(3), 4)
    b = 3 + np.tile(np.arange(4), 3)
    lay, L = sp.layer_assign(a, b, 7)
    assert L == 2 and _valid(a, b, lay)
    a = np.arange(5)
    b = (a + 1) % 5
    lay, L = sp.layer_assign(a, b, 5)
    assert L == 3 and _valid(a, b, lay)
    lay, L = sp.layer_assign([], [], 0)
    assert L == 0 and len(lay) == 0


def test_random_graphs_valid_and_greedy_bound():
    rng = np.random.default_rng(11)
    for trial in range(30):
        P = int(rng.integers(1, 300))
        m = int(rng.integers(0, 4 * P))
        a = rng.integers(0, P, m)
        b = rng.integers(0, P, m)
        lay, L = sp.layer_assign(np.concatenate([a, np.arange(P)]), np.concatenate([b, np.arange(P)]), P)  # + self pairs
        assert _valid(a, b, lay)
        assert lay.min() >= 0 and lay.max() == L - 1
        deg = np.zeros(P, np.int64)
        ne = a != b
        pairs = {(min(x, y), max(x, y)) for x, y in zip(a[ne], b[ne])}
        for x, y in pairs:
            deg[x] += 1
            deg[y] += 1
        assert L <= (deg.max() if P else 0) + 1
        lay2, L2 = sp.layer_assign(np.concatenate([a, np.arange(P)]), np.concatenate([b, np.arange(P)]), P)
        assert L2 == L and np.array_equal(lay2, lay)          # deterministic


def test_bad_arguments():
    with pytest.raises(sp.SpadeError):
        sp.layer_assign([0], [5], 3)
    with pytest.raises(sp.SpadeError):
        sp.layer_assign([-1], [0], 3)
