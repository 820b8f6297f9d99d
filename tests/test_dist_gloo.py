"""World-size-2 CPU (gloo) tests of the multi-GPU protocol of fgr_route_all.

The device path (include/fastgr.h, fgr_route_all with a communicator) does, per
batch: split the batch by tree edges with fgr_split_batch, route the rank's chunk
into zero-padded route records, SUM-all-reduce the records, then commit every net
of the batch from the records; a batch of fewer than split_min nets is routed whole
on every rank with no exchange.  Here the same protocol runs on CPU with gloo, the
split taken from the library's host-only fgr_split_batch and the per-net routing
from the oracle; the result must equal the single-process oracle bit for bit
(nets of one batch are independent: reading R13).  The library's own exchange path
(split arithmetic, record offsets, partial launches, commit from records) runs on
one GPU under fgr_set_exchange's emulated ranks: tests/test_gpu_exchange.py.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
from oracle import Oracle
from paper_conf_date_liulzclly22_b200 import fastgr as F


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def batch_order(d, b, nb):
    """Nets grouped by batch, larger nets first (the library's exec order), then id."""
    sizes = d.net_sizes()
    out = []
    for bb in range(nb):
        ids = np.nonzero(b == bb)[0]
        ids = sorted(ids, key=lambda n: (-sizes[n], n))
        out.append(np.array(ids, np.int64))
    return out


def _worker(rank, world, port, cfg, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        d = cfg()
        o = Oracle(d)
        b, nb = o.plan()
        # the plan is replicated: every rank must hold the same batches
        h = torch.tensor([int(np.int64(b.astype(np.int64) @ np.arange(1, len(b) + 1)) % (1 << 61)), nb])
        hs = [torch.zeros_like(h) for _ in range(world)]
        dist.all_gather(hs, h)
        assert all(torch.equal(x, h) for x in hs)
        sizes = d.net_sizes()
        demand = o.zero_demand()
        seg = np.zeros(d.num_nodes, np.uint32)
        cost = np.zeros(d.num_nets, np.uint32)
        for n in range(d.num_nets):
            if sizes[n] == 1:
                seg[d.node_offset[n]] = 0xFFFFFFFF
        for bb, ids in enumerate(batch_order(d, b, nb)):
            nl = int((sizes[ids] > 32).sum())
            ep = np.concatenate([[0], np.cumsum(sizes[ids] - 1)])
            l0, l1, s0, s1, whole = F.fgr_split_batch(len(ids), nl, rank, world, ep, SPLIT_MIN)
            if whole:   # routed whole on every rank, no exchange
                assert (l0, l1, s0, s1) == (0, nl, nl, len(ids))
                for n in ids:
                    s_, c_ = o.route_net(int(n), demand)
                    a, e = d.node_offset[n], d.node_offset[n + 1]
                    seg[a:e] = s_[a:e]
                    cost[n] = c_
                for n in ids:
                    o.commit_net(int(n), seg, demand)
                continue
            mine = list(ids[l0:l1]) + list(ids[s0:s1])
            rec = np.zeros(d.num_nodes, np.int64)
            rc = np.zeros(d.num_nets, np.int64)
            for n in mine:
                s_, c_ = o.route_net(int(n), demand)
                a, e = d.node_offset[n], d.node_offset[n + 1]
                rec[a:e] = s_[a:e]
                rc[n] = c_
            t = torch.from_numpy(rec)
            tc = torch.from_numpy(rc)
            dist.all_reduce(t, op=dist.ReduceOp.SUM)
            dist.all_reduce(tc, op=dist.ReduceOp.SUM)
            recs = t.numpy().astype(np.uint32)
            for n in ids:
                a, e = d.node_offset[n], d.node_offset[n + 1]
                seg[a:e] = recs[a:e]
                cost[n] = np.uint32(tc.numpy()[n])
                o.commit_net(int(n), seg, demand)
        q.put((rank, seg.tobytes(), cost.tobytes(), demand.tobytes()))
    finally:
        dist.destroy_process_group()


SPLIT_MIN = 20   # small enough that tiny/t1 exercise both the split and the whole-batch path


def _run(cfg, world=2):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, cfg, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return sorted(res)


def _cfg_tiny():
    return gen.make_config("tiny")


def _cfg_t1():
    return gen.make_config("t1", num_nets=1500)


def _cfg_big():
    return gen.generate(nx=80, ny=80, nlayers=6, num_nets=150, seed=31, caps=[1, 3, 3, 3, 3, 3], pin_dist=1,
                        kmin=10, kmax=120, hpwl_base=12.0, hpwl_sigma=0.5, name="bigmix")


@pytest.mark.parametrize("cfg", [_cfg_tiny, _cfg_t1, _cfg_big], ids=["tiny", "t1", "bigmix"])
def test_two_rank_exchange_equals_single_process(cfg):
    d = cfg()
    o = Oracle(d)
    b, nb = o.plan()
    seg1, cost1, dem1 = o.route(b, nb)
    res = _run(cfg, world=2)
    for rank, seg, cost, dem in res:
        assert np.array_equal(np.frombuffer(seg, np.uint32), seg1), rank
        assert np.array_equal(np.frombuffer(cost, np.uint32), cost1), rank
        assert np.array_equal(np.frombuffer(dem, np.int32).reshape(dem1.shape), dem1), rank


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_split_covers_batch(world):
    rng = np.random.default_rng(world)
    for _ in range(200):
        count = int(rng.integers(0, 500))
        nl = int(rng.integers(0, count + 1))
        seen = []
        for r in range(world):
            l0, l1, s0, s1, whole = F.fgr_split_batch(count, nl, r, world)
            assert whole == 0
            assert 0 <= l0 <= l1 <= nl <= s0 <= s1 <= count
            seen += list(range(l0, l1)) + list(range(s0, s1))
            assert abs((l1 - l0) - nl / world) <= 1 and abs((s1 - s0) - (count - nl) / world) <= 1
        assert sorted(seen) == list(range(count))
    with pytest.raises(F.FgrError):
        F.fgr_split_batch(10, 11, 0, 1)


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_split_balances_tree_edges(world):
    """Edge-balanced split: covering, and each rank's share of the large
    (small) nets' edges is within one net's edges of the ideal."""
    rng = np.random.default_rng(10 + world)
    for _ in range(200):
        count = int(rng.integers(1, 400))
        nl = int(rng.integers(0, count + 1))
        edges = np.concatenate([np.sort(rng.integers(33, 1000, size=nl))[::-1], rng.integers(1, 32, size=count - nl)])
        ep = np.concatenate([[0], np.cumsum(edges)])
        seen = []
        for r in range(world):
            l0, l1, s0, s1, whole = F.fgr_split_batch(count, nl, r, world, ep, 0)
            assert whole == 0 and 0 <= l0 <= l1 <= nl <= s0 <= s1 <= count
            seen += list(range(l0, l1)) + list(range(s0, s1))
            el = edges[:nl].sum() / world
            es = edges[nl:].sum() / world
            assert abs(edges[l0:l1].sum() - el) <= (edges[:nl].max() if nl else 0)
            assert abs(edges[s0:s1].sum() - es) <= (edges[nl:].max() if count > nl else 0)
        assert sorted(seen) == list(range(count))
        for r in range(world):   # below split_min: every rank takes the whole batch
            assert F.fgr_split_batch(count, nl, r, world, ep, count + 1) == (0, nl, nl, count, 1)
