"""Pins for the oracle's RNG, permutation and rank partition (O1-O3).

O1 Philox4x32-10 is pinned to Random123's published known-answer vectors
(tests/golden/philox4x32_10_kat.txt); bounded()/bern() to their closed-form
bucket boundaries; O2 to the permutation property and to uniformity over all
n! orders; O3 exactly to torch.utils.data.DistributedSampler(shuffle=False)
(north_star: "sharded by clip in DistributedSampler order") and to the
exactly-once rule.
"""
import math
import os
from itertools import permutations

import numpy as np
import pytest
import scipy.stats

import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden", "philox4x32_10_kat.txt")


def _kat():
    rows = []
    for line in open(GOLD):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        v = [int(t, 16) for t in line.split()]
        rows.append((v[0:4], v[4:6], v[6:10]))
    return rows


@pytest.mark.parametrize("ctr,key,expect", _kat())
def test_philox_known_answer(ctr, key, expect):
    assert oracle.philox(ctr, key) == expect


def test_philox_counter_sensitivity():
    # every counter word and key word changes the output (a dropped word would not)
    base = oracle.philox([1, 2, 3, 4], [5, 6])
    for i in range(4):
        c = [1, 2, 3, 4]
        c[i] ^= 1
        assert oracle.philox(c, [5, 6]) != base
    for i in range(2):
        k = [5, 6]
        k[i] ^= 1
        assert oracle.philox([1, 2, 3, 4], k) != base


@pytest.mark.parametrize("n", [1, 2, 3, 5, 7, 10, 224, 1000, 65537, 2**31 + 1, 2**32 - 1])
def test_bounded_bucket_boundaries(n):
    # floor(x*n/2^32) == k exactly on [ceil(k 2^32/n), ceil((k+1) 2^32/n)): check both edges
    ks = sorted({0, 1, n // 2, n - 1} | set(range(min(n, 40))))
    for k in ks:
        if k >= n:
            continue
        lo = -(-(k << 32) // n)
        assert oracle.bounded(lo, n) == k
        if k > 0:
            assert oracle.bounded(lo - 1, n) == k - 1
    assert oracle.bounded(0, n) == 0
    assert oracle.bounded(2**32 - 1, n) == n - 1


def test_bounded_exact_bucket_counts_small_n():
    # exact bucket sizes over all 2^32 inputs follow from the boundaries above
    for n in (3, 5, 7):
        sizes = [(-(-((k + 1) << 32) // n)) - (-(-(k << 32) // n)) for k in range(n)]
        assert sum(sizes) == 2**32
        assert max(sizes) - min(sizes) <= 1


def test_bern_thresholds():
    assert oracle.bern(0, 0.0) == 0 and oracle.bern(2**32 - 1, 0.0) == 0
    assert oracle.bern(0, 1.0) == 1 and oracle.bern(2**32 - 1, 1.0) == 1
    assert oracle.bern(2**31 - 1, 0.5) == 1 and oracle.bern(2**31, 0.5) == 0
    assert oracle.bern(2**30 - 1, 0.25) == 1 and oracle.bern(2**30, 0.25) == 0


def test_u01_exact():
    L = oracle.lib()
    assert L.oracle_u01(0) == 0.0
    assert L.oracle_u01(2**31) == 0.5
    assert L.oracle_u01(2**32 - 1) == (2**32 - 1) / 2**32


@pytest.mark.parametrize("n", [1, 2, 3, 10, 97, 1024])
def test_permutation_is_permutation(n):
    for e in range(5):
        p = oracle.permutation(n, seed=1234, epoch=e)
        assert sorted(p.tolist()) == list(range(n))


def test_permutation_deterministic_and_epoch_dependent():
    a = oracle.permutation(1024, 7, 3)
    b = oracle.permutation(1024, 7, 3)
    c = oracle.permutation(1024, 7, 4)
    d = oracle.permutation(1024, 8, 3)
    assert (a == b).all()
    assert (a != c).any() and (a != d).any()


@pytest.mark.parametrize("n", [3, 4])
def test_permutation_uniform_over_all_orders(n):
    # chi-square over all n! orders (Fisher-Yates with an unbiased draw is uniform)
    orders = {p: i for i, p in enumerate(permutations(range(n)))}
    trials = 600 * len(orders)
    counts = np.zeros(len(orders))
    for e in range(trials):
        counts[orders[tuple(oracle.permutation(n, seed=99, epoch=e).tolist())]] += 1
    stat, p = scipy.stats.chisquare(counts)
    assert p > 1e-5, (counts, p)


@pytest.mark.parametrize("n,world", [(10, 1), (10, 3), (12, 4), (7, 8), (1024, 8), (5, 2), (3, 5), (100, 7)])
@pytest.mark.parametrize("drop_last", [False, True])
def test_partition_matches_torch_distributed_sampler(n, world, drop_last):
    from torch.utils.data import DistributedSampler
    perm = oracle.permutation(n, seed=5, epoch=2)
    for rank in range(world):
        s = DistributedSampler(list(range(n)), num_replicas=world, rank=rank, shuffle=False,
                               drop_last=drop_last)
        expect = [int(perm[i]) for i in s]
        got = oracle.partition(perm, world, rank, drop_last).tolist()
        assert got == expect
        assert oracle.lib().oracle_num_samples(n, world, int(drop_last)) == len(s)


@pytest.mark.parametrize("n,world", [(1024, 8), (1024, 4), (1024, 1), (96, 3)])
def test_partition_exactly_once_per_epoch(n, world):
    # "Each video must be processed and used exactly once per epoch"
    perm = oracle.permutation(n, seed=11, epoch=0)
    allc = np.concatenate([oracle.partition(perm, world, r, False) for r in range(world)])
    assert sorted(allc.tolist()) == list(range(n))


def test_permutation_epoch_high_bits_enter_the_key():
    # R#1: the counter holds the epoch's low word; its high word is XORed into the
    # key's high word, so epochs e and e + 2^32 are independent streams and the stream of
    # (seed, e + 2^32) is the one of (seed ^ 2^32, e)
    a = oracle.permutation(1024, 7, 3)
    b = oracle.permutation(1024, 7, 3 + 2**32)
    c = oracle.permutation(1024, 7 ^ (1 << 32), 3)
    assert (a != b).any()
    assert (b == c).all()
