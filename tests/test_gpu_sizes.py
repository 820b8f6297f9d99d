"""Large-net size boundaries of the DP kernels, bit-exact against the oracle: random trees of
exactly 127/128/129 nodes (k_dp_tree 128-thread / 256-thread variants), 511/512/513 (256 /
384-thread variants) and the shared-memory capacity of the 384-thread variant and beyond (the
nets above it take k_dp_hld).  Random recursive trees (parent[j] < j, reading R22) with random
pin spans (R4) and no zero-length edges (R8); one net per batch position so that several size
classes run in the same batch."""
import numpy as np
import pytest

import gen
from oracle import Oracle
from tests.test_gpu_parity import first_diff

pytestmark = pytest.mark.gpu


def random_tree_design(sizes, seed, n=400, L=9):
    rng = np.random.default_rng(seed)
    xs, ys, plo, phi, par, off = [], [], [], [], [], [0]
    for k, m in enumerate(sizes):
        cx, cy = rng.integers(60, n - 60, 2)
        x = np.zeros(m, np.int64); y = np.zeros(m, np.int64); p = np.full(m, -1, np.int64)
        x[0], y[0] = cx, cy
        for j in range(1, m):
            u = int(rng.integers(0, j))
            p[j] = u
            while True:   # a short edge from the parent, never zero-length, inside the grid
                dx, dy = rng.integers(-6, 7, 2)
                if rng.random() < 0.3:
                    dy = 0   # straight edges too (reading R7)
                if (dx or dy) and 0 <= x[u] + dx < n and 0 <= y[u] + dy < n:
                    break
            x[j], y[j] = x[u] + dx, y[u] + dy
        lo = np.full(m, -1, np.int64); hi = np.full(m, -1, np.int64)
        pin = rng.random(m) < 0.6
        lo[pin] = rng.integers(0, 2, pin.sum()); hi[pin] = lo[pin] + rng.integers(0, 3, pin.sum())
        xs.append(x); ys.append(y); plo.append(lo); phi.append(hi); par.append(p); off.append(off[-1] + m)
    cat = lambda a, t: np.concatenate(a).astype(t)
    return gen.Design(nx=n, ny=n, nlayers=L, dir=np.array([l % 2 for l in range(L)], np.uint8),
                      layer_capacity=np.array(gen.CAP9[:L], np.int32), edge_capacity=None,
                      node_offset=np.array(off, np.int32), x=cat(xs, np.int16), y=cat(ys, np.int16),
                      pin_lo=cat(plo, np.int8), pin_hi=cat(phi, np.int8), parent=cat(par, np.int32),
                      name="sizes", seed=seed)


@pytest.mark.parametrize("sizes,seed", [
    ([127, 128, 129, 33, 64, 65], 1),
    ([511, 512, 513, 256, 257], 2),
    ([1040, 1055, 1056, 1057, 1100, 1200], 3),
])
def test_size_boundaries_bit_exact(sizes, seed):
    from paper_conf_date_liulzclly22_b200 import Router
    d = random_tree_design(sizes, seed)
    r = Router(d, device=0)
    r.reset_demand(None)
    nb = r.plan()
    r.route_all()
    b, nb, seg, cost, dem = r.results()
    o = Oracle(d)
    ob, onb = o.plan()
    assert nb == onb and np.array_equal(b, ob)
    oseg, ocost, odem = o.route(ob, onb)
    assert np.array_equal(seg, oseg), first_diff(seg, oseg)
    assert np.array_equal(cost, ocost), first_diff(cost, ocost)
    assert np.array_equal(dem, odem), first_diff(dem.ravel(), odem.ravel())
    r.close()
