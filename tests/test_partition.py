"""Multi-GPU sharding: the native LPT partition against a plain Python LPT
and its guarantees (every index exactly once, deterministic, imbalance <= the largest item)."""
import heapq

import numpy as np
import pytest

import vbgen
from paper_conf_ipps_abdelfattahhtd16_b200 import shard, vbatched_partition_lpt


def _lpt_py(n, g):
    order = sorted(range(len(n)), key=lambda i: (-int(n[i]), i))
    loads = [0.0] * g
    owner = [0] * len(n)
    for i in order:
        r = min(range(g), key=lambda k: (loads[k], k))
        owner[i] = r
        loads[r] += float(n[i]) ** 3 / 3.0
    return np.array(owner, dtype=np.int32)


@pytest.mark.parametrize("g", [1, 2, 3, 4, 8])
def test_native_lpt_matches_python(g):
    n = vbgen.sizes("C3")[:700]
    assert np.array_equal(vbatched_partition_lpt(n, g) if g > 1 else shard.lpt_owner(n, g),
                          _lpt_py(n, g))


@pytest.mark.parametrize("g", [2, 4, 8])
def test_lpt_balance_c5(g):
    n = vbgen.sizes("C5")
    owner = shard.lpt_owner(n, g)
    assert owner.min() == 0 and owner.max() == g - 1
    loads = shard.shard_loads(n, g)
    big = float(n.max()) ** 3 / 3.0
    assert loads.max() - loads.min() <= big
    assert (loads.max() - loads.min()) / loads.mean() < 1e-3  # < 0.1 % at C5
    idx = np.concatenate([shard.shard_indices(n, g, r) for r in range(g)])
    assert np.array_equal(np.sort(idx), np.arange(len(n)))


def test_partition_deterministic_and_argument_checks():
    n = vbgen.sizes("C4")
    assert np.array_equal(vbatched_partition_lpt(n, 4), vbatched_partition_lpt(n.copy(), 4))
    from paper_conf_ipps_abdelfattahhtd16_b200 import lib
    assert lib().vbatched_partition_lpt(n.ctypes.data, len(n), 0, n.ctypes.data) == -3
