"""Host-side logic of libsmoothe.so, no GPU needed: the C ABI loads and
exports every symbol include/smoothe.h declares, and the e-graph loader's
derived quantities (de-duplicated E, SCC partition, K_auto, error codes)
agree with the independent fp64 oracle's analysis."""
import ctypes
import os
import re

import numpy as np
import pytest

from gen import make_config, random_tiny

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def sm():
    import paper_conf_asplos_caiydyz25_b200 as pkg
    if not os.path.exists(pkg.smoothe.LIB_PATH):
        import __graft_entry__
        __graft_entry__.build()
    pkg.lib()
    return pkg


def header_functions():
    src = open(os.path.join(ROOT, "include", "smoothe.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(smoothe_[a-z_]+)\s*\(", src)))


def test_exports_every_declared_symbol(sm):
    names = header_functions()
    assert len(names) >= 15
    L = ctypes.CDLL(sm.smoothe.LIB_PATH)
    for n in names:
        assert hasattr(L, n), n
    assert set(names) == set(sm.smoothe._SIGS), "binding and header disagree"
    assert "sm_100a" in sm.version()


def test_only_abi_symbols_exported(sm):
    import subprocess
    out = subprocess.run(["nm", "-D", "--defined-only", sm.smoothe.LIB_PATH], capture_output=True,
                         text=True).stdout
    syms = [l.split()[-1] for l in out.splitlines() if " T " in l]
    ours = [s for s in syms if s.startswith("smoothe_")]
    assert set(ours) == set(header_functions())


def _host_graph(sm, eg):
    return sm.load_egraph(eg.class_ptr, eg.child_ptr, eg.child_class, eg.root, device=-1)


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C5"])
def test_loader_matches_oracle_analysis(sm, orc, name):
    eg = make_config(name)
    g = _host_graph(sm, eg)
    o = orc.Graph(eg)
    assert g.info["num_edges"] == o.E
    assert g.info["K_auto"] == o.K_auto
    assert g.info["num_scc"] == o.num_scc
    assert g.info["scc_classes"] == o.scc_classes
    assert g.info["scc_max"] == o.scc_max
    assert g.info["device"] == -1
    a, b = g.scc(), o.scc()
    assert np.array_equal(a >= 0, b >= 0)
    # same partition: a relabelling
    pairs = {(x, y) for x, y in zip(a, b) if x >= 0}
    assert len(pairs) == len({x for x, _ in pairs}) == len({y for _, y in pairs})


@pytest.mark.parametrize("p_back", [0.06, 0.15])
def test_loader_large_components(sm, orc, p_back):
    # components above 64 classes (the global-memory penalty / decode paths)
    eg = make_config("C2", scc_max=10**9, p_back=p_back)
    g = _host_graph(sm, eg)
    o = orc.Graph(eg)
    assert g.info["scc_max"] == o.scc_max > 64
    assert (g.info["num_scc"], g.info["scc_classes"], g.info["K_auto"]) == \
        (o.num_scc, o.scc_classes, o.K_auto)


def test_loader_tiny_families(sm, orc):
    for s in range(60):
        eg = random_tiny(2000 + s, ["tree", "dag", "cyclic"][s % 3])
        g = _host_graph(sm, eg)
        o = orc.Graph(eg)
        assert (g.info["num_edges"], g.info["K_auto"], g.info["num_scc"]) == (o.E, o.K_auto, o.num_scc)


def test_duplicate_children_are_removed(sm):
    # root {r -> A, A, B}; A {a}; B {b}
    g = sm.load_egraph([0, 1, 2, 3], [0, 3, 3, 3], [1, 1, 2], 0, device=-1)
    assert g.info["num_edges"] == 2


@pytest.mark.parametrize("bad,code", [
    (dict(class_ptr=[0, 1, 1, 3]), "E_BAD_GRAPH"),          # empty class (S28)
    (dict(child_class=[1, 7]), "E_BAD_GRAPH"),              # child id out of range
    (dict(root=5), "E_BAD_GRAPH"),                          # root out of range
    (dict(class_ptr=[0, 2, 1, 3]), "E_BAD_GRAPH"),          # not monotone
    (dict(child_ptr=[0, 2, 1, 2]), "E_BAD_GRAPH"),          # child_ptr not monotone
])
def test_loader_rejects_bad_graphs(sm, bad, code):
    args = dict(class_ptr=[0, 1, 2, 3], child_ptr=[0, 2, 2, 2], child_class=[1, 2], root=0)
    args.update(bad)
    with pytest.raises(sm.SmootheError) as ei:
        sm.load_egraph(args["class_ptr"], args["child_ptr"], args["child_class"], args["root"], device=-1)
    assert code in str(ei.value)


def test_host_only_graph_cannot_run(sm):
    eg = make_config("C1")
    g = _host_graph(sm, eg)
    with pytest.raises(sm.SmootheError) as ei:
        sm.run_create(g, sm.CostModel.from_input(eg), 1)
    assert "E_STATE" in str(ei.value)


def test_product_package_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_asplos_caiydyz25_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h", ".cuh", "Makefile")):
                txt = open(os.path.join(dirpath, f)).read().lower()
                assert "oracle" not in txt, f"{f} mentions the oracle"
