"""The Gbase-style comparison join (gsh_join_gbase; §II-B,
§III): no skew handling, R sub-lists against the full S partition, chained shared-memory
table, write-bitmap output rounds.  It computes the same equi-join, so it must equal the oracle
bit-exactly (count, checksum, sorted pairs) like GSH."""
import numpy as np
import pytest
import torch

import datagen
import oracle
import paper_conf_icde_caic24_b200 as gsh

pytestmark = pytest.mark.gpu
DEV = "cuda"


def _np(t):
    return t.cpu().numpy().view(np.uint32)


def _dev(*ts):
    return [t.to(DEV) for t in ts]


def _sorted_pairs(p):
    a = p.cpu().numpy().view(np.uint32).reshape(-1, 2)
    return a[np.lexsort((a[:, 1], a[:, 0]))]


@pytest.mark.parametrize("kind,n,theta", [("uniform", 100_000, 0.0), ("pkfk", (1 << 18) + 5, 0.0),
                                          ("zipf", 1 << 18, 0.5), ("zipf", (1 << 16) + 7, 0.75),
                                          ("zipf", 1 << 16, 1.0), ("zipf", 1 << 14, 1.5),
                                          ("graph", 1 << 16, 0.909), ("pkfk_zipf", 1 << 17, 1.0),
                                          ("uniform", 3, 0.0)])
def test_gbase_count_checksum(kind, n, theta):
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=19)
    on, oc, _ = oracle.join(_np(rk), _np(rp), _np(sk), _np(sp))
    r = gsh.join(*_dev(rk, rp, sk, sp), impl="gbase", config=gsh.make_config(timing=True))
    assert (r.count, r.checksum) == (on, oc)
    st = r.stats
    assert st["n_heavy"] == 0 and st["ms_nmjoin"] > 0


@pytest.mark.parametrize("kind,n,theta", [("zipf", 40_000, 1.0), ("pkfk", 100_003, 0.0), ("graph", 1 << 15, 0.909)])
def test_gbase_materialize_pairs_exact(kind, n, theta):
    rk, rp, sk, sp = datagen.make_workload(kind, n, theta, seed=5)
    on, oc, op = oracle.join_sorted_pairs(_np(rk), _np(rp), _np(sk), _np(sp))
    r = gsh.join(*_dev(rk, rp, sk, sp), mode="materialize", out_capacity=on + 10, impl="gbase")
    assert (r.count, r.checksum, r.written, r.overflow) == (on, oc, on, False)
    assert np.array_equal(_sorted_pairs(r.pairs), op)


def test_gbase_overflow_subset_and_config():
    rk, rp, sk, sp = datagen.zipf_pair(30_000, 30_000, 1.0, seed=8)
    on, oc, _ = oracle.join(_np(rk), _np(rp), _np(sk), _np(sp))
    d = _dev(rk, rp, sk, sp)
    r = gsh.join(*d, mode="materialize", out_capacity=on // 3, impl="gbase")
    assert (r.count, r.checksum, r.written, r.overflow) == (on, oc, on // 3, True)
    got = _sorted_pairs(r.pairs)
    assert np.all(_np(rk)[got[:, 0]] == _np(sk)[got[:, 1]])
    assert np.unique(got, axis=0).shape[0] == got.shape[0]
    for cfg in (dict(pass_bits=(3, 2)), dict(pass_bits=(0, 0)), dict(hybrid=True)):
        r = gsh.join(*d, impl="gbase", config=gsh.make_config(**cfg))
        assert (r.count, r.checksum) == (on, oc)


def test_gbase_edge_cases():
    z = torch.zeros
    cases = [(z(9000, dtype=torch.int32), torch.arange(9000, dtype=torch.int32),   # one key, 3 sub-lists
              z(700, dtype=torch.int32), torch.arange(700, dtype=torch.int32)),
             (z(0, dtype=torch.int32), z(0, dtype=torch.int32), z(10, dtype=torch.int32),
              torch.arange(10, dtype=torch.int32)),
             (torch.full((5,), -1, dtype=torch.int32), torch.arange(5, dtype=torch.int32),
              torch.tensor([-1, 0], dtype=torch.int32), torch.arange(2, dtype=torch.int32))]
    for rk, rp, sk, sp in cases:
        on, oc, op = oracle.join_sorted_pairs(_np(rk), _np(rp), _np(sk), _np(sp))
        m = gsh.join(*_dev(rk, rp, sk, sp), mode="materialize", out_capacity=on, impl="gbase")
        assert (m.count, m.checksum, m.written) == (on, oc, on)
        assert np.array_equal(_sorted_pairs(m.pairs), op)
