"""The Vose alias table the GPU builds by a MERGE (csrc/pf_kernels.cuh
resample_group, csrc/pf_central.cu vz_merge) equals the sequential sweep of
reading R10 (the oracle, oracle/orc_impl.inc) — checked here in plain Python
on random weights, ties and degenerate cases, with the same merge-path
partitioning into P outputs per thread.  (The GPU tables themselves are
compared with the oracle bit for bit in tests/test_gpu_parity.py and
tests/test_gpu_central.py.)"""
import numpy as np
import pytest


def merge_table(q, T):
    """prob / alias by one merge of A (exclusive deficits over the small
    slots) and E (inclusive excesses over the large slots), A first on ties;
    T threads, each: one diagonal search + P = M / T merge steps."""
    M = len(q)
    P = M // T
    Q = int(q.sum())
    a = [M * int(x) for x in q]
    L = [s for s in range(M) if a[s] < Q]
    H = [s for s in range(M) if a[s] >= Q]
    nL, nH = len(L), len(H)
    A, acc = [], 0
    for s in L:
        A.append(acc)
        acc += Q - a[s]
    Dtot = acc
    E, acc = [], 0
    for s in H:
        acc += a[s] - Q
        E.append(acc)
    prob, alias = [None] * M, [None] * M
    for t in range(T):
        diag = t * P
        lo, hi = max(0, diag - nH), min(diag, nL)
        while lo < hi:
            mid = (lo + hi) // 2
            if A[mid] <= E[diag - 1 - mid]:
                lo = mid + 1
            else:
                hi = mid
        i, j = lo, diag - lo
        Ai = A[i] if i < nL else Dtot
        Bj = E[j] if j < nH else 1 << 64
        for _ in range(P):
            if i < nL and Ai <= Bj:
                s = L[i]
                An = A[i + 1] if i + 1 < nL else Dtot
                pr, al = Q - (An - Ai), H[j]
                i, Ai = i + 1, An
            else:
                s = H[j]
                pr, al = (Q + Bj - Ai, H[j + 1]) if Bj < Dtot else (Q, s)
                j += 1
                Bj = E[j] if j < nH else 1 << 64
            assert prob[s] is None
            prob[s], alias[s] = pr, al
    return np.array(prob, np.uint64), np.array(alias, np.int32)


def _weights(rng, M, kind):
    if kind == "uniform":
        q = np.full(M, 1 << 22)
    elif kind == "onehot":
        q = np.zeros(M, np.int64)
        q[rng.integers(0, M)] = 1 << 22
    elif kind == "ties":
        q = rng.integers(0, 4, M) * (1 << 20)
        q[0] = 1 << 22
    elif kind == "sparse":
        q = np.where(rng.random(M) < 0.5, 0, rng.integers(0, 1 << 22, M))
        q[rng.integers(0, M)] = 1 << 22
    else:
        q = np.floor(np.exp(-rng.exponential(4, M)) * (1 << 22)).astype(np.int64)
        q[rng.integers(0, M)] = 1 << 22
    return q.astype(np.uint32)


@pytest.mark.parametrize("kind", ["uniform", "onehot", "ties", "sparse", "decay"])
def test_merge_equals_sweep(orc, kind):
    rng = np.random.default_rng(hash(kind) % 1000)
    for _ in range(40):
        M = int(rng.choice([32, 64, 128, 256, 512, 1024]))
        T = int(rng.choice([t for t in (32, 64, 128, 256) if t <= M]))
        q = _weights(rng, M, kind)
        p, a = merge_table(q, T)
        po, ao = orc.vose_build(q)
        np.testing.assert_array_equal(p, po)
        np.testing.assert_array_equal(a, ao)


def test_golden_table(orc):
    # SURVEY §8(c) golden vector: q = [4, 1, 0, 3] -> prob [4, 4, 0, 8], alias [3, 0, 0, 3]
    p, a = merge_table(np.array([4, 1, 0, 3], np.uint32), 1)
    assert p.tolist() == [4, 4, 0, 8] and a.tolist() == [3, 0, 0, 3]
