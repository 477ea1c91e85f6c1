"""GPU parity of the layer index (spade_build_layered / spade_join_count_layered; PAPER.md P:148,
P:200): per-polygon COUNT through one probe pass per layer must equal the brute-force
oracle and the single owner-set canvas, bit for bit; the layers must be valid (no two polygons of a
layer intersect: checked against the polygon x polygon join) and cover every polygon once."""
import numpy as np
import pytest

import gen
import oracle
from gen import configs
from tests.helpers import lattice, valid_polyset

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def spade():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_icde_doraiswamyf22_b200 as sp
    sp.load()
    return sp


def _layers_valid(sp, polys, lc):
    a, b = sp.join_polygons(polys, polys)
    a, b = a.cpu().numpy(), b.cpu().numpy()
    lay = lc.layer_of()
    ne = a != b
    assert np.all(lay[a[ne]] != lay[b[ne]])
    assert lay.min() >= 0 and lay.max() == lc.num_layers - 1


@pytest.mark.parametrize("seed", range(4))
def test_layered_count_matches_oracle_on_overlapping_valid_sets(spade, seed):
    import torch
    rng = np.random.default_rng(900 + seed)
    polys = valid_polyset(rng, int(rng.integers(8, 40)), 0, 48)
    xy = lattice(-2, -2, 50, 50)
    lc = spade.LayeredCanvas(polys, max_dim=int(rng.choice([16, 64, 512])))
    assert lc.num_layers >= 1
    _layers_valid(spade, polys, lc)
    got = spade.join_count_layered(lc, torch.as_tensor(xy).cuda()).cpu().numpy()
    np.testing.assert_array_equal(got, oracle.join_count(xy, polys))
    cv = spade.Canvas(polys, max_dim=64)
    np.testing.assert_array_equal(got, spade.join_count(cv, torch.as_tensor(xy).cuda()).cpu().numpy())


def test_layered_count_on_overlapping_stars(spade):
    """A reduced ov workload (stars piled over the point clusters): layered COUNT == owner-set COUNT
    over 2M points, and == the oracle on a sample of them."""
    import torch
    w = configs.ov(n_points=2_000_000, n_polys=120)
    lc = spade.LayeredCanvas(w.polys, max_dim=w.max_dim)
    _layers_valid(spade, w.polys, lc)
    assert lc.num_layers > 1
    xy = gen.points_device(w.points, w.point_seed, 0, w.n_points)
    got = spade.join_count_layered(lc, xy).cpu().numpy()
    ref = spade.join_count(spade.Canvas(w.polys, max_dim=w.max_dim), xy).cpu().numpy()
    np.testing.assert_array_equal(got, ref)
    idx = np.random.default_rng(5).integers(0, w.n_points, 20000)
    xs = gen.points_at(w.points, w.point_seed, idx)
    sub = spade.join_count_layered(lc, torch.as_tensor(xs).cuda()).cpu().numpy()
    np.testing.assert_array_equal(sub, oracle.join_count(xs, w.polys))
