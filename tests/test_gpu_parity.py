"""GPU parity: the CUDA path through the C ABI vs. the CPU oracle, element by element.

Bar (north_star): batch membership, per-segment (bend, ls, lt,
straight), per-net cost and the final demand grid are bit-exact.  Inputs are the
seeded synthetic designs of gen/ (recipe in DESIGN.md §4).
"""
import numpy as np
import pytest

import gen
from oracle import Oracle

pytestmark = pytest.mark.gpu


def _router(d):
    from paper_conf_date_liulzclly22_b200 import Router
    return Router(d, device=0)


def first_diff(a, b):
    idx = np.nonzero(a != b)[0]
    return None if len(idx) == 0 else (int(idx[0]), a[idx[0]], b[idx[0]], len(idx))


def check_against_oracle(d, r=None, demand0=None):
    import torch
    own = r is None
    if own:
        r = _router(d)
    if demand0 is not None:
        r.reset_demand(torch.from_numpy(demand0).cuda())
    else:
        r.reset_demand(None)
    nb = r.plan()
    r.route_all()
    b, nb, seg, cost, dem = r.results()
    o = Oracle(d)
    ob, onb = o.plan()
    assert nb == onb, (nb, onb)
    assert np.array_equal(b, ob), first_diff(b, ob)
    oseg, ocost, odem = o.route(ob, onb, demand=demand0)
    assert np.array_equal(seg, oseg), first_diff(seg, oseg)
    assert np.array_equal(cost, ocost), first_diff(cost, ocost)
    assert np.array_equal(dem, odem), first_diff(dem.ravel(), odem.ravel())
    if own:
        r.close()
    return nb


@pytest.mark.parametrize("cfg", ["tiny", "t1", "t5"])
def test_configs_bit_exact(cfg):
    nb = check_against_oracle(gen.make_config(cfg))
    assert nb > 1


@pytest.mark.parametrize("seed", range(12))
def test_random_small_bit_exact(seed):
    L = [2, 3, 4, 5, 6, 9, 12, 16][seed % 8]
    d = gen.random_small(seed=90 + seed, nx=40 + 7 * seed, ny=33 + 5 * seed, nlayers=L, num_nets=300,
                         kmax=12, literal_frac=0.3, caps=[1] + [2] * (L - 1))
    check_against_oracle(d)


def test_nonuniform_directions_and_costs():
    d = gen.random_small(seed=5, nx=50, ny=60, nlayers=7, num_nets=400, kmax=9)
    d.dir = np.array([1, 1, 0, 1, 0, 0, 1], np.uint8)   # not alternating, V first
    rng = np.random.default_rng(1)
    d.via_cost = rng.integers(0, 90, size=6).astype(np.int32)
    d.ovf_weight = rng.integers(0, 9000, size=7).astype(np.int32)
    d.len_cost = 17
    d.logistic_slope = 0.37
    d.slack_clamp = 9
    check_against_oracle(d)


def test_initial_demand_and_edge_capacity():
    d = gen.make_config("t1", num_nets=1500)
    rng = np.random.default_rng(2)
    d.edge_capacity = rng.integers(0, 12, size=(d.nlayers, d.ny, d.nx)).astype(np.uint8)
    dem0 = rng.integers(0, 9, size=(d.nlayers, d.ny, d.nx)).astype(np.int32)
    # unused entries (last column of H layers, last row of V layers) are ignored by both sides
    for l in range(d.nlayers):
        if d.dir[l] == 0:
            dem0[l, :, -1] = 0
        else:
            dem0[l, -1, :] = 0
    check_against_oracle(d, demand0=dem0)


def test_big_nets_cta_path():
    """Nets with > 32 nodes take the one-CTA-per-net path."""
    d = gen.generate(nx=120, ny=110, nlayers=9, num_nets=400, seed=77, caps=gen.CAP9, pin_dist=1, kmin=30,
                     kmax=400, hpwl_base=20.0, hpwl_sigma=0.5, name="bignets")
    assert (d.net_sizes() > 32).sum() > 100
    check_against_oracle(d)


@pytest.mark.parametrize("L", [3, 5, 12, 16])
def test_big_nets_layer_counts(L):
    """The flow (33..64 nodes by default) and heavy-path (> 64 nodes) kernels at other layer counts:
    L <= 15 backtracks through tabulated span maps, L = 16 through the scalar span walk."""
    caps = [2] + [6] * (L - 1)
    d = gen.generate(nx=90, ny=80, nlayers=L, num_nets=150, seed=300 + L, caps=caps, pin_dist=1, kmin=20,
                     kmax=300, hpwl_base=18.0, hpwl_sigma=0.5, literal_frac=0.2, name=f"big{L}")
    sizes = d.net_sizes()
    assert ((sizes > 32) & (sizes <= 128)).sum() > 10 and (sizes > 128).sum() > 5
    check_against_oracle(d)


def test_route_batch_matches_oracle_batches():
    import torch
    d = gen.make_config("t1")
    o = Oracle(d)
    ob, onb = o.plan()
    oseg, ocost, odem = o.route(ob, onb)
    r = _router(d)
    r.reset_demand(None)
    r.seg.fill_(-1)
    r.cost.zero_()
    for b in range(onb):
        ids = torch.from_numpy(np.nonzero(ob == b)[0].astype(np.int32)).cuda()
        r.route_batch(ids)
    torch.cuda.synchronize()
    seg = r.seg.cpu().numpy().view(np.uint32)
    cost = r.cost.cpu().numpy().view(np.uint32)
    assert np.array_equal(seg, oseg), first_diff(seg, oseg)
    assert np.array_equal(cost, ocost)
    assert np.array_equal(r.demand().cpu().numpy(), odem)
    r.close()


def test_repeat_runs_identical_and_demand_roundtrip():
    import torch
    d = gen.make_config("tiny")
    r = _router(d)
    r.run()
    a = r.results()
    r.run()
    b = r.results()
    for x, y in zip(a, b):
        assert np.array_equal(np.asarray(x), np.asarray(y))
    dem = torch.randint(0, 50, (d.nlayers, d.ny, d.nx), dtype=torch.int32, device="cuda")
    for l in range(d.nlayers):
        if d.dir[l] == 0:
            dem[l, :, -1] = 0
        else:
            dem[l, -1, :] = 0
    r.reset_demand(dem)
    assert torch.equal(r.demand(), dem)
    r.close()


def test_edge_cases_empty_and_trivial():
    d = gen.make_config("tiny", num_nets=0)
    r = _router(d)
    r.run()
    b, nb, seg, cost, dem = r.results()
    assert nb == 0 and dem.sum() == 0
    r.close()
    # only single-node (trivial) nets
    d1 = gen.make_config("tiny", num_nets=50)
    keep = [n for n in range(d1.num_nets)]
    t = d1.subset(keep)
    first = t.node_offset[:-1]
    t2 = gen.Design(t.nx, t.ny, t.nlayers, t.dir, t.layer_capacity, None, np.arange(len(first) + 1, dtype=np.int32),
                    t.x[first], t.y[first], t.pin_lo[first], t.pin_hi[first], np.full(len(first), -1, np.int32))
    r = _router(t2)
    r.run()
    b, nb, seg, cost, dem = r.results()
    assert nb == 0 and np.all(b == -1) and np.all(seg == 0xFFFFFFFF) and np.all(cost == 0) and dem.sum() == 0
    r.close()


def test_invalid_nets_rejected():
    from paper_conf_date_liulzclly22_b200 import FgrError
    d = gen.make_config("tiny", num_nets=30)
    a = d.node_offset[7]
    d.parent = d.parent.copy()
    d.parent[a + 1] = 5 if d.node_offset[8] - a > 1 else d.parent[a + 1]
    r = _router(d)
    with pytest.raises(FgrError) as e:
        r.plan()
    assert e.value.status == 1 and "net 7" in str(e.value)
    r.close()
    d = gen.make_config("tiny", num_nets=30)
    d.x = d.x.copy()
    a = d.node_offset[3]
    d.x[a + 1] = d.x[a + d.parent[a + 1]]
    d.y = d.y.copy()
    d.y[a + 1] = d.y[a + d.parent[a + 1]]          # zero-length edge
    r = _router(d)
    with pytest.raises(FgrError):
        r.plan()
    r.close()


def test_t9_full_size_bit_exact():
    """BASELINE.json's headline config at full size (~900k nets), as bench.py runs it."""
    check_against_oracle(gen.make_config("t9"))


def test_scale_full_size_bit_exact():
    """BASELINE.json configs[4] (2M nets, 2000 x 2000, 9 layers) at full size: the
    largest design the library routes, every net, batch and demand cell compared."""
    check_against_oracle(gen.make_config("scale"))


@pytest.mark.parametrize("cfg", ["tiny", "t5"])
def test_exchange_path_world1_bit_exact(cfg):
    """The multi-GPU path (split -> route records -> NCCL all-reduce -> commit from
    records) run with a world-1 NCCL communicator on one GPU."""
    from paper_conf_date_liulzclly22_b200 import fastgr as F
    d = gen.make_config(cfg)
    r = _router(d)
    F.fgr_comm_init(r.h, F.fgr_comm_unique_id(), 0, 1)
    check_against_oracle(d, r=r)
    st = F.fgr_get_stats(r.h)
    assert st["world"] == 1
    r.close()
