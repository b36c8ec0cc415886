"""Oracle pins: exchange topology and the particle exchange (Algorithm 2
l.10–14; Fig.1; §VI-E; readings R2–R5, R19)."""
import json
import os

import numpy as np

from conftest import GOLDEN

G = json.load(open(os.path.join(GOLDEN, "exchange_golden.json")))


def test_neighbor_tables_by_hand(orc):
    ring = orc.Config(m=4, n_filters=4, t=1, topo="ring")
    assert [orc.neighbors(ring, n) for n in range(4)] == G["ring"]["neighbors"]
    tor = orc.Config(m=8, n_filters=4, t=1, topo="torus")
    assert orc.torus_shape(tor) == (2, 2)
    assert [orc.neighbors(tor, n) for n in range(4)] == G["torus"]["neighbors"]
    assert orc.neighbors(orc.Config(topo="none"), 3) == []


def test_torus_default_shape(orc):
    # R = 2^floor(log2(N)/2), C = N/R (R4)
    for N, RC in [(16, (4, 4)), (4096, (64, 64)), (65536, (256, 256)), (2048, (32, 64)), (8, (2, 4))]:
        assert orc.torus_shape(orc.Config(n_filters=N, topo="torus")) == RC


def test_torus_neighbors_wrap(orc):
    cfg = orc.Config(n_filters=12, topo="torus", torus_rows=3, torus_cols=4)
    # sub-filter 0 at (0,0): up (2,0)=8, down (1,0)=4, left (0,3)=3, right (0,1)=1
    assert orc.neighbors(cfg, 0) == [8, 4, 3, 1]
    assert orc.neighbors(cfg, 11) == [7, 3, 10, 8]
    # symmetric: q is a neighbour of n iff n is a neighbour of q
    for n in range(12):
        for q in orc.neighbors(cfg, n):
            assert n in orc.neighbors(cfg, q)


def test_exchange_golden_ring(orc):
    g = G["ring"]
    cfg = orc.Config(m=g["m"], n_filters=g["N"], t=g["t"], topo="ring")
    np.testing.assert_array_equal(orc.exchange(cfg, g["logw"]), g["src"])


def test_exchange_golden_torus(orc):
    g = G["torus"]
    cfg = orc.Config(m=g["m"], n_filters=g["N"], t=g["t"], topo="torus")
    np.testing.assert_array_equal(orc.exchange(cfg, g["logw"]), g["src"])


def test_exchange_t0_and_none_is_identity(orc, W):
    w = W.random_logw(8, 32, 2)
    ident = np.arange(8 * 32).reshape(8, 32)
    np.testing.assert_array_equal(orc.exchange(orc.Config(m=32, n_filters=8, t=0, topo="ring"), w), ident)
    np.testing.assert_array_equal(orc.exchange(orc.Config(m=32, n_filters=8, t=2, topo="none"), w), ident)


def test_exchange_properties_brute_force(orc, W):
    # on random sets with ties: exactly deg*t slots change per sub-filter, they
    # are the deg*t worst by (logw desc, slot asc), and they receive, in order,
    # the t best of each neighbour
    for topo, N, m, t in [("ring", 6, 16, 3), ("torus", 16, 32, 2), ("ring", 2, 8, 1), ("torus", 4, 64, 4)]:
        cfg = orc.Config(m=m, n_filters=N, t=t, topo=topo)
        w = W.random_logw(N, m, N + m + t)
        src = orc.exchange(cfg, w)
        rank = lambda n: sorted(range(m), key=lambda i: (-w[n][i], i))
        for n in range(N):
            nb = orc.neighbors(cfg, n)
            deg = len(nb)
            worst = rank(n)[::-1][:deg * t]
            incoming = [q * m + rank(q)[j] for q in nb for j in range(t)]
            for j, slot in enumerate(worst):
                assert src[n][slot] == incoming[j]
            for slot in set(range(m)) - set(worst):
                assert src[n][slot] == n * m + slot


def test_exchange_golden_all2all(orc):
    g = G["all2all"]
    for t, key in [(1, "src_t1"), (2, "src_t2")]:
        cfg = orc.Config(m=g["m"], n_filters=g["N"], t=t, topo="all2all")
        np.testing.assert_array_equal(orc.exchange(cfg, g["logw"]), g[key])


def test_all2all_brute_force(orc, W):
    # every sub-filter's worst t slots receive the global best t of the pool
    # of supplied particles (each sub-filter's best t), in order
    for N, m, t in [(8, 16, 3), (5, 32, 1), (16, 8, 2)]:
        cfg = orc.Config(m=m, n_filters=N, t=t, topo="all2all")
        w = W.random_logw(N, m, N * m + t)
        src = orc.exchange(cfg, w)
        rank = lambda n: sorted(range(m), key=lambda i: (-w[n][i], i))
        pool = [n * m + rank(n)[j] for n in range(N) for j in range(t)]
        top = sorted(pool, key=lambda p: (-w.ravel()[p], p))[:t]
        for n in range(N):
            worst = rank(n)[::-1][:t]
            for j, slot in enumerate(worst):
                assert src[n][slot] == top[j]
            for slot in set(range(m)) - set(worst):
                assert src[n][slot] == n * m + slot
