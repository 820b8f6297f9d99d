"""CPU-only checks of the C ABI: the library loads, exports every symbol the header
declares, and its host-side cost table equals the oracle's (reading R1/R18)."""
import ctypes
import re
import os

import numpy as np
import pytest

import gen
from oracle import Oracle
from paper_conf_date_liulzclly22_b200 import fastgr as F

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    src = open(os.path.join(ROOT, "include", "fastgr.h")).read()
    return sorted(set(re.findall(r"FGR_API\s+[\w\s\*]+?\b(fgr_\w+)\s*\(", src)))


def test_header_symbols_exported():
    syms = header_symbols()
    assert len(syms) >= 14
    lib = ctypes.CDLL(F.LIB_PATH)
    for s in syms:
        assert hasattr(lib, s), s
    assert sorted(F.EXPORTS) == syms


def test_version_and_error_string():
    assert "sm_100a" in F.fgr_version()
    assert isinstance(F.lib().fgr_last_error(), bytes)


@pytest.mark.parametrize("cfg", ["tiny", "t1"])
def test_cost_table_matches_oracle(cfg):
    d = gen.make_config(cfg, num_nets=10)
    desc = F.make_desc(d.nx, d.ny, d.nlayers, d.dir, d.layer_capacity, d.len_cost, d.via_cost, d.ovf_weight,
                       d.logistic_slope, d.slack_clamp)
    assert np.array_equal(F.fgr_cost_table(desc), Oracle(d).cost_table())


def test_cost_table_other_params():
    d = gen.make_config("tiny", num_nets=1)
    rng = np.random.default_rng(3)
    for _ in range(5):
        d.ovf_weight = rng.integers(0, 100000, size=d.nlayers).astype(np.int32)
        d.logistic_slope = float(rng.uniform(0.1, 3.0))
        d.slack_clamp = int(rng.integers(1, 200))
        desc = F.make_desc(d.nx, d.ny, d.nlayers, d.dir, d.layer_capacity, d.len_cost, d.via_cost, d.ovf_weight,
                           d.logistic_slope, d.slack_clamp)
        assert np.array_equal(F.fgr_cost_table(desc), Oracle(d).cost_table())


def test_desc_validation_errors():
    d = gen.make_config("tiny", num_nets=1)
    bad = F.make_desc(d.nx, d.ny, d.nlayers, np.zeros(d.nlayers, np.uint8), d.layer_capacity, d.len_cost,
                      d.via_cost, d.ovf_weight, d.logistic_slope, d.slack_clamp)
    with pytest.raises(F.FgrError) as e:
        F.fgr_cost_table(bad)
    assert e.value.status == F.FGR_ERR_INVALID
    big = F.make_desc(30000, 30000, d.nlayers, d.dir, d.layer_capacity, d.len_cost, d.via_cost,
                      np.full(d.nlayers, 1 << 20, np.int32), d.logistic_slope, d.slack_clamp)
    with pytest.raises(F.FgrError) as e:
        F.fgr_cost_table(big)
    assert e.value.status == F.FGR_ERR_RANGE


def test_no_cpu_fallback_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(RuntimeError):
        F.Router(gen.make_config("tiny", num_nets=5))


def test_setters_reject_null_grid():
    """Host-only setters validate their grid argument without a device (FGR_ERR_INVALID)."""
    lib = F.lib()
    assert lib.fgr_set_graph(None, 1) == F.FGR_ERR_INVALID
    assert lib.fgr_set_exchange(None, 16, 0) == F.FGR_ERR_INVALID
    assert lib.fgr_set_dp_policy(None, 0, 64) == F.FGR_ERR_INVALID
