"""Host logic of the balanced chunks (uc_balance_plan), no device: the table is a
partition of every strip's rows into its chunks in order, respects the minimum chunk sizes the
kernel needs (a non-edge chunk never reaches a halo row), deals blocks to strips so the strips'
summed rates match, sizes chunks in proportion to rates, and equal rates give the static layout."""
import numpy as np
import pytest

import paper_conf_cluster_sagbilieinu25_b200 as U


def _valid(tab, strips, chunks, n, shrink, levels):
    assert tab.shape == (strips * chunks, 4)
    assert sorted(map(tuple, tab[:, :2].tolist())) == [(s, q) for s in range(strips) for q in range(chunks)]
    for s in range(strips):
        rows = sorted((r[1], r[2], r[3]) for r in tab if r[0] == s)
        assert rows[0][1] == 1 and rows[-1][2] == n
        for (q0, lo0, hi0), (q1, lo1, hi1) in zip(rows, rows[1:]):
            assert lo1 == hi0 + 1
        if chunks > 1:
            assert rows[0][2] >= levels + 2            # chunk 1 starts below row levels + 1
            assert n - rows[-1][1] + 1 >= levels + 2   # the last but one ends above n - levels
            for q, lo, hi in rows[1:-1]:
                assert hi - lo + 1 >= levels


@pytest.mark.parametrize("strips,chunks,n,shrink,levels", [(21, 14, 16384, 160, 8), (6, 49, 2048, 30, 8),
                                                           (3, 1, 40, 0, 8), (4, 2, 100, 20, 6), (1, 5, 90, 0, 4)])
def test_equal_rates_give_the_static_layout(strips, chunks, n, shrink, levels):
    tab = U.balance_plan(strips, chunks, n, shrink, levels)
    _valid(tab, strips, chunks, n, shrink, levels)
    b = np.arange(strips * chunks)
    assert np.array_equal(tab[:, 0], b % strips) and np.array_equal(tab[:, 1], b // strips)
    E = n + 2 * shrink
    for r in tab:  # the static chunking's cuts, up to rounding
        q = r[1]
        lo_static = 1 + max(0, min(q * E // chunks - shrink, n))
        assert abs(r[2] - lo_static) <= 1


@pytest.mark.parametrize("seed", range(5))
def test_random_rates_partition_and_balance(seed):
    rng = np.random.default_rng(seed)
    strips, chunks, n, shrink, levels = 21, 14, 16384, 160, 8
    rates = rng.choice([1.0, 1.16, 1.28], strips * chunks) * rng.uniform(0.98, 1.02, strips * chunks)
    tab = U.balance_plan(strips, chunks, n, shrink, levels, rates)
    _valid(tab, strips, chunks, n, shrink, levels)
    sums = np.array([rates[tab[:, 0] == s].sum() for s in range(strips)])
    assert sums.max() / sums.min() < 1.01          # strips carry equal summed rates (LPT)
    # rows in proportion to rates: every block's predicted march time within 2 % of its strip's
    E = n + 2 * shrink
    for s in range(strips):
        sel = np.nonzero(tab[:, 0] == s)[0]
        eff = tab[sel, 3] - tab[sel, 2] + 1 + np.where((tab[sel, 1] == 0) | (tab[sel, 1] == chunks - 1), shrink, 0)
        t = eff / rates[sel]
        assert t.max() / t.min() < 1.02
        assert eff.sum() == E


def test_extreme_rates_keep_minimum_sizes():
    strips, chunks, n, shrink, levels = 3, 8, 300, 20, 8
    rates = np.array([1e-6, 1e6] * (strips * chunks // 2))
    tab = U.balance_plan(strips, chunks, n, shrink, levels, rates)
    _valid(tab, strips, chunks, n, shrink, levels)


def test_too_few_rows_is_an_error():
    with pytest.raises(Exception):
        U.balance_plan(2, 10, 50, 0, 8)
