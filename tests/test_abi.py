"""C-ABI checks that need no GPU: the library loads, exports every symbol that
include/*.h declares, and the host-only planner behaves as DESIGN.md states."""
import ctypes
import glob
import os
import re

import pytest

import oracle as O
import tdfs_inputs as T
import paper_conf_icde_yuan0ha0024_b200 as M
from tests.test_oracle import AUT

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_symbols():
    names = set()
    for h in glob.glob(os.path.join(ROOT, "include", "*.h")):
        src = open(h).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        src = re.sub(r"//[^\n]*", "", src)
        for m in re.finditer(r"\b(tdfs_[a-z0-9_]+)\s*\(", src):
            names.add(m.group(1))
    return sorted(names)


def test_library_exports_every_declared_symbol():
    lib = ctypes.CDLL(M.LIB_PATH)
    names = _declared_symbols()
    assert len(names) >= 20
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing
    # and the binding wraps every one of them
    assert set(names) <= set(M.SIGNATURES), set(names) - set(M.SIGNATURES)


def test_library_is_sm100a():
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", M.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_abi_version_and_status_strings():
    assert M.tdfs_abi_version() == 2
    assert M.tdfs_status_string(0) == "TDFS_OK"
    assert M.tdfs_status_string(8) == "TDFS_E_STACK_EXHAUSTED"
    o = M.default_opts()
    assert o.tau_ns == 10_000_000 and o.chunk == 8 and o.queue_ints == 3_000_000 and o.page_bytes == 8192


@pytest.mark.parametrize("name", sorted(AUT))
def test_planner_aut_and_constraints_match_oracle(name):
    q = T.query(name)
    p = M.plan_from_query(q)
    assert p.aut_size() == AUT[name]
    n_aut, cons = O.automorphisms(q)
    assert sorted(p.constraints()) == sorted(cons)


def test_planner_greedy_order_rule():
    # first = highest degree (lowest id on ties); then most placed neighbours, higher degree, lower id
    assert M.plan_from_query(T.query("triangle")).order() == [0, 1, 2]
    assert M.plan_from_query(T.query("diamond")).order() == [1, 2, 0, 3]
    assert M.plan_from_query(T.query("house")).order() == [0, 1, 4, 2, 3]
    assert M.plan_from_query(T.query("tailed_triangle")).order() == [2, 0, 1, 3]
    assert M.plan_from_query(T.query("w5")).order()[0] == 0  # the hub
    for name in AUT:
        q = T.query(name)
        order = M.plan_from_query(q).order()
        assert sorted(order) == list(range(q.k))
        adj = {(a, b) for a, b in q.edges} | {(b, a) for a, b in q.edges}
        for i in range(1, q.k):
            assert any((order[i], order[j]) in adj for j in range(i)), (name, order)


def test_planner_overrides_and_errors():
    q = T.query("fig1_q")
    p = M.plan_from_query(q, order=[0, 2, 1, 3, 4], constraints=[(0, 2)])
    assert p.order() == [0, 2, 1, 3, 4] and p.constraints() == [(0, 2)]
    assert M.plan_from_query(q, constraints="none").constraints() == []
    with pytest.raises(M.TdfsError) as e:
        M.plan_from_query(q, order=[0, 4, 1, 2, 3])  # u5 not adjacent to u1
    assert e.value.status == M.TDFS_E_QUERY_DISCONNECTED
    with pytest.raises(M.TdfsError) as e:
        M.tdfs_plan_query(9, [(i, i + 1) for i in range(8)])
    assert e.value.status == M.TDFS_E_QUERY_TOO_LARGE
    with pytest.raises(M.TdfsError) as e:
        M.tdfs_plan_query(3, [(0, 1), (1, 2)], qlabel=[0, 300, 1])
    assert e.value.status == M.TDFS_E_LABEL_RANGE
    with pytest.raises(M.TdfsError) as e:
        M.tdfs_plan_query(3, [(0, 1)])
    assert e.value.status == M.TDFS_E_QUERY_DISCONNECTED
    with pytest.raises(M.TdfsError) as e:
        M.tdfs_plan_query(3, [(0, 0), (1, 2)])
    assert e.value.status == M.TDFS_E_INVALID_ARG
    with pytest.raises(M.TdfsError) as e:
        M.tdfs_plan_query(3, [(0, 1), (1, 2)], order=[0, 0, 1])
    assert e.value.status == M.TDFS_E_INVALID_ARG


def test_labeled_planner_aut():
    q = T.labeled_query("c4", 2)   # labels 0,1,0,1 -> Aut = rotations by 2 and reflections preserving labels
    p = M.plan_from_query(q)
    assert p.aut_size() == O.automorphisms(q)[0] == 4
