"""CPU-only checks of the product library: it loads, exports every symbol that
include/gsword.h declares, and its host-side logic (graph canonical check, query
plan compilation, HT finalisation) behaves as the header documents.  No compute
call is made without a GPU."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_journals_pacmmod_yelsg24_b200 as G
from paper_journals_pacmmod_yelsg24_b200 import gsword as binding
from gsword_testutil import ROOT, read_golden
from workloads import gen


def _declared_symbols():
    src = open(os.path.join(ROOT, "include", "gsword.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gsword_[a-z_0-9]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    syms = _declared_symbols()
    assert len(syms) >= 15
    lib = ctypes.CDLL(binding.LIB_PATH)
    for s in syms:
        assert hasattr(lib, s), s


def test_version():
    assert G.version() == 200


def test_check_graph_accepts_canonical(c0):
    g, _ = c0
    G.check_graph(g.row_ptr, g.col, g.labels, g.n_labels)
    G.check_graph(gen.ring_graph(9).row_ptr, gen.ring_graph(9).col)


@pytest.mark.parametrize("mutation,status", [
    ("self_loop", -5), ("unsorted", -5), ("asymmetric", -5), ("out_of_range", -5), ("bad_label", -1),
    ("labels_null_multi", -1), ("row_ptr0", -5),
])
def test_check_graph_rejects(mutation, status):
    g = gen.random_small_graph(12, 0.4, 3, seed=4)
    rp, col, lab, nl = g.row_ptr.copy(), g.col.copy(), g.labels.copy(), 3
    v = int(np.argmax(np.diff(rp)))
    if mutation == "self_loop":
        col[rp[v]] = v
        col[rp[v]:rp[v + 1]] = np.sort(col[rp[v]:rp[v + 1]])
    elif mutation == "unsorted":
        col[rp[v]], col[rp[v] + 1] = col[rp[v] + 1], col[rp[v]]
    elif mutation == "asymmetric":
        # drop one direction of an edge
        w = int(col[rp[v]])
        keep = np.ones(col.shape[0], bool)
        keep[rp[v]] = False
        col = col[keep]
        rp = rp.copy()
        rp[v + 1:] -= 1
    elif mutation == "out_of_range":
        col[rp[v + 1] - 1] = 12
    elif mutation == "bad_label":
        lab[3] = 3
    elif mutation == "labels_null_multi":
        lab = None
    elif mutation == "row_ptr0":
        rp = rp.copy()
        rp[0] = 1
    with pytest.raises(G.GswordError) as e:
        G.check_graph(rp, col, lab, nl)
    assert e.value.status == status


def test_plan_query_masks():
    # query: 0-1, 1-2, 2-0, 2-3 (paw); labels 0,1,0,0; order 2,0,1,3
    q = gen.query_from_edges(4, [(0, 1), (1, 2), (2, 0), (2, 3)], labels=[0, 1, 0, 0], order=[2, 0, 1, 3])
    p = G.plan_query(*q.csr(), q.labels, q.order, 2)
    assert p["label"] == [0, 0, 1, 0]
    # B(1) = {0} (0-2 edge); B(2) = {0,1} (1-2, 1-0); B(3) = {0} (3-2)
    assert p["back_mask"] == [0, 0b1, 0b11, 0b1]
    # same-label earlier positions: d1 (label0): {0}; d2 (label1): {}; d3 (label0): {0,1}
    assert p["dup_mask"] == [0, 0b1, 0, 0b11]


def test_plan_query_errors():
    q = gen.path_query(3)
    with pytest.raises(G.GswordError) as e:
        G.plan_query(*q.csr(), q.labels, [0, 2, 1], 1)  # prefix {0,2} disconnected
    assert e.value.status == -4
    with pytest.raises(G.GswordError) as e:
        G.plan_query(*q.csr(), q.labels, [0, 0, 1], 1)
    assert e.value.status == -4
    with pytest.raises(G.GswordError) as e:
        G.plan_query(*q.csr(), [0, 0, 5], q.order, 2)
    assert e.value.status == -1
    big = gen.path_query(17)
    with pytest.raises(G.GswordError) as e:
        G.plan_query(*big.csr(), big.labels, big.order, 1)
    assert e.value.status == -6
    # asymmetric query CSR
    with pytest.raises(G.GswordError) as e:
        G.plan_query([0, 1, 1], [1], [0, 0], [0, 1], 1)
    assert e.value.status == -1


def test_finalize_example2():
    # Ex. 2: samples {0, 24} -> sum 24, sumsq 576, 1 valid of 2 -> estimate 12
    r = G.finalize([24.0, 576.0, 1.0, 2.0])
    assert r["estimate"] == 12.0 and r["n"] == 2 and r["n_valid"] == 1
    assert r["variance"] == pytest.approx((576 - 24 * 24 / 2) / 2, rel=1e-15)


def test_qerror_golden():
    for c, ch, want in read_golden("qerror_cases.txt"):
        assert G.qerror(float(c), float(ch)) == pytest.approx(float(want), rel=1e-15)


def test_no_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    with pytest.raises(G.GswordError) as e:
        G.Context(0)
    assert e.value.status == -7


def test_product_package_does_not_touch_oracle():
    pkg = os.path.join(ROOT, "paper_journals_pacmmod_yelsg24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
                src = open(os.path.join(dirpath, f)).read()
                assert "oracle" not in src.replace("CPU oracle", ""), f


def test_quicksi_order_golden():
    rows = {r[0]: r[1:] for r in read_golden("quicksi_example.txt")}
    labels = np.array([int(x) for x in rows["ex1_labels"]], np.int32)
    e = [tuple(int(y) for y in x.split("-")) for x in rows["ex1_edges"]]
    g = gen.make_graph(labels.shape[0], [a for a, _ in e], [b for _, b in e], labels, 3)
    qe = [tuple(int(y) for y in x.split("-")) for x in rows["ex1_qedges"]]
    q = gen.query_from_edges(4, qe, labels=[int(x) for x in rows["ex1_qlabels"]], order=[0, 1, 2, 3])
    qrp, qcol = q.csr()
    assert G.quicksi_order(g.row_ptr, g.col, g.labels, 3, qrp, qcol, q.labels) == [int(x) for x in rows["ex1_order"]]
    ring = gen.ring_graph(10)
    p4 = gen.path_query(4)
    qrp, qcol = p4.csr()
    assert G.quicksi_order(ring.row_ptr, ring.col, None, 1, qrp, qcol, p4.labels) == [int(x) for x in rows["ex2_order"]]


@pytest.mark.parametrize("seed", range(10))
def test_quicksi_order_valid(seed):
    g = gen.random_small_graph(15, 0.3, 3, seed=seed)
    q = gen.random_connected_query(2 + seed % 10, 0.3, 3, seed)
    qrp, qcol = q.csr()
    order = G.quicksi_order(g.row_ptr, g.col, g.labels, 3, qrp, qcol, q.labels)
    assert sorted(order) == list(range(q.nq))
    p = G.plan_query(qrp, qcol, q.labels, order, 3)  # raises EORDER unless every prefix is connected
    assert p["nq"] == q.nq
