"""Pins the closed-form labelled-star count used by scripts/sweep_c4.py
against brute force."""
import os
import sys

import pytest

from oracle import exact
from workloads import gen

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "scripts"))
from sweep_c4 import star_count  # noqa: E402


@pytest.mark.parametrize("seed", range(8))
def test_star_closed_form(seed):
    g = gen.random_small_graph(9, 0.5, 1 + seed % 3, seed=3000 + seed)
    s = 2 + seed % 3
    q = gen.star_query_from(g, s, seed) if (g.degree() >= s).any() else gen.star_query(2, [0, 0, 0])
    assert star_count(g, int(q.labels[0]), [int(x) for x in q.labels[1:]]) == exact.brute_force_count(g, q)


def test_c4_small_scale_builds():
    g, qs = gen.config_c4(scale=12, n_edges=20_000, sizes=(4, 6))
    assert g.n == 4096 and g.n_edges == 20_000 and g.n_labels == 16
    assert [q.nq for q in qs] == [4, 4, 6, 6, 4, 5, 6]
