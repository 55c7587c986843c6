"""Skeleton planning (pure host logic, no GPU) against the structure the
paper gives for its Fig. 4a example — axpy (map) -> laplace (stencil) ->
dot (reduce) — in PAPER.md §V (L279-L396):
  * the data dependency graph: RaW / WaR edges, only the stencil incoherent
    (it needs a halo update on X), L284-L290;
  * the multi-GPU graph: a halo node before the stencil, the map -> dot
    dependency removed as redundant (L296-L299); Standard OCC splits the
    stencil, Extended also the map, Two-way also the reduce with an internal
    -> boundary reduce dependency (L304-L316); hints launch the internal
    stencil and internal reduce before the halo (L318-L330);
  * the schedule: BFS levels, parent-stream reuse, an event per
    cross-stream dependency, task order by BFS over data + hints
    (L352-L396)."""
import pytest

import paper_conf_ipps_meneghinmjm22_b200 as nb

X, Y = 0, 1
FIG4A = [(nb.SK_AXPBY, Y, X, 0.125, 1.0, 0),  # x <- x + a y   (map)
         (nb.SK_LAPLACE7, X, Y, 0.0, 0.0, 0),  # y <- L(x)      (stencil, halo on X)
         (nb.SK_DOT, X, Y, 0.0, 0.0, 0)]       # <x, y>         (reduce)


def plan(nparts, occ, containers=FIG4A):
    return nb.nb_skeleton_plan(nparts, occ, containers)


def by_name(p):
    return {n["name"]: n for n in p["nodes"]}


def edges(p, key="data"):
    names = {n["id"]: n["name"] for n in p["nodes"]}
    return {(names[a], names[b]) for a, b in p[key]}


def check_schedule(p):
    """order is topological for data + hints; every cross-stream data edge
    has an event the child waits on; same-stream edges are enqueued in order."""
    pos = {u: i for i, u in enumerate(p["order"])}
    assert sorted(p["order"]) == list(range(len(p["nodes"])))
    for a, b in p["data"] + p["hints"]:
        assert pos[a] < pos[b]
    nodes = p["nodes"]
    for a, b in p["data"]:
        if nodes[a]["stream"] != nodes[b]["stream"]:
            assert nodes[a]["event"] >= 0 and nodes[a]["event"] in nodes[b]["waits"]
    for n in nodes:
        assert 0 <= n["stream"] < p["streams"]
    levels = {}
    for n in nodes:
        levels.setdefault(n["level"], []).append(n)
    for a, b in p["data"]:
        assert nodes[a]["level"] < nodes[b]["level"]


def test_no_occ_graph_matches_fig4b_4c():
    p = plan(2, nb.OCC_NONE)
    names = [n["name"] for n in p["nodes"]]
    assert names == ["axpby#0", "halo(f0)", "laplace7#1", "dot#2"]
    n = by_name(p)
    assert [n[k]["op"] for k in names] == ["map", "halo", "stencil", "reduce"]
    assert all(n[k]["view"] == "standard" for k in names)
    # only the stencil is incoherent (it reads X's halo)
    assert [k for k in names if n[k]["incoherent"]] == ["laplace7#1"]
    # map -> halo -> stencil -> dot; the direct map -> dot dependency (dot reads
    # X) is transitively implied and removed as redundant
    assert edges(p) == {("axpby#0", "halo(f0)"), ("halo(f0)", "laplace7#1"), ("laplace7#1", "dot#2")}
    # one compute stream plus the transfer stream; the chain needs the two
    # cross-stream events around the halo
    assert p["streams"] == 2 and p["events"] == 2
    check_schedule(p)


def test_single_partition_needs_no_halo_and_no_split():
    for occ in (nb.OCC_NONE, nb.OCC_STANDARD, nb.OCC_EXTENDED, nb.OCC_TWO_WAY):
        p = plan(1, occ)
        assert [n["name"] for n in p["nodes"]] == ["axpby#0", "laplace7#1", "dot#2"]
        assert not any(n["incoherent"] for n in p["nodes"])
        check_schedule(p)


def test_standard_occ_splits_the_stencil_and_overlaps_the_halo():
    p = plan(2, nb.OCC_STANDARD)
    n = by_name(p)
    assert set(n) == {"axpby#0", "halo(f0)", "laplace7#1[int]", "laplace7#1[bnd]", "dot#2"}
    e = edges(p)
    assert ("axpby#0", "halo(f0)") in e and ("halo(f0)", "laplace7#1[bnd]") in e
    assert ("axpby#0", "laplace7#1[int]") in e
    # the internal stencil does not wait for the halo: concurrent, on another
    # stream, launched first (hint)
    assert ("halo(f0)", "laplace7#1[int]") not in e
    assert n["halo(f0)"]["stream"] != n["laplace7#1[int]"]["stream"]
    assert ("laplace7#1[int]", "halo(f0)") in edges(p, "hints")
    check_schedule(p)


def test_extended_occ_splits_the_map_feeding_the_stencil():
    p = plan(2, nb.OCC_EXTENDED)
    n = by_name(p)
    assert {"axpby#0[bnd]", "axpby#0[int]"} <= set(n)
    e = edges(p)
    # the halo needs only the boundary map; internal map + internal stencil overlap it
    assert ("axpby#0[bnd]", "halo(f0)") in e and ("axpby#0[int]", "halo(f0)") not in e
    assert ("axpby#0[int]", "laplace7#1[int]") in e
    hints = edges(p, "hints")
    assert ("axpby#0[int]", "halo(f0)") in hints and ("laplace7#1[int]", "halo(f0)") in hints
    assert "dot#2" in n  # the reduce after the stencil is not split
    check_schedule(p)


def test_two_way_occ_splits_the_reduce_with_internal_before_boundary():
    p = plan(2, nb.OCC_TWO_WAY)
    n = by_name(p)
    assert {"dot#2[int]", "dot#2[bnd]"} <= set(n)
    assert n["dot#2[bnd]"]["finalize"] and not n["dot#2[int]"]["finalize"]
    e = edges(p)
    assert ("dot#2[int]", "dot#2[bnd]") in e  # the added internal -> boundary dependency
    assert ("laplace7#1[int]", "dot#2[int]") in e and ("laplace7#1[bnd]", "dot#2[bnd]") in e
    hints = edges(p, "hints")
    # the two hints of Fig. 4d (internal stencil, internal reduce) — plus the
    # internal map, which is also concurrent with the transfer here
    assert {("laplace7#1[int]", "halo(f0)"), ("dot#2[int]", "halo(f0)")} <= hints
    # the halo has a stream of its own, so the hinted internal work never
    # queues in front of it
    assert sum(1 for x in p["nodes"] if x["stream"] == n["halo(f0)"]["stream"]) == 1
    order = [p["nodes"][u]["name"] for u in p["order"]]
    assert order.index("dot#2[int]") < order.index("halo(f0)") < order.index("laplace7#1[bnd]")
    check_schedule(p)


def test_loop_of_ten_iterations_and_coherency():
    c1 = []
    for k in range(10):
        c1 += [(nb.SK_AXPBY, Y, X, 0.125, 1.0, 0), (nb.SK_LAPLACE7, X, Y, 0, 0, 0), (nb.SK_DOT, X, Y, 0, 0, k)]
    for occ in (nb.OCC_NONE, nb.OCC_STANDARD, nb.OCC_EXTENDED, nb.OCC_TWO_WAY):
        p = plan(4, occ, c1)
        assert sum(n["op"] == "halo" for n in p["nodes"]) == 10  # X rewritten every iteration
        check_schedule(p)
    # two stencils reading X with no write in between share one halo update
    p = plan(2, nb.OCC_STANDARD, [(nb.SK_LAPLACE7, X, Y, 0, 0, 0), (nb.SK_LAPLACE7, X, 2, 0, 0, 0)])
    assert sum(n["op"] == "halo" for n in p["nodes"]) == 1
    # a map writing the stencil's output makes nothing incoherent for X
    p = plan(2, nb.OCC_NONE, [(nb.SK_LAPLACE7, X, Y, 0, 0, 0), (nb.SK_AXPBY, 2, Y, 1, 1, 0),
                              (nb.SK_LAPLACE7, X, 3, 0, 0, 0)])
    assert sum(n["op"] == "halo" for n in p["nodes"]) == 1


def test_reductions_serialise_on_the_shared_scratch_and_slots():
    c = [(nb.SK_DOT, X, X, 0, 0, 0), (nb.SK_DOT, Y, Y, 0, 0, 1)]
    p = plan(2, nb.OCC_TWO_WAY, c)
    assert edges(p) == {("dot#0", "dot#1")}


def test_invalid_plans_fail():
    with pytest.raises(nb.NbError):
        plan(2, nb.OCC_NONE, [(nb.SK_LAPLACE7, X, X, 0, 0, 0)])  # in place stencil
    with pytest.raises(nb.NbError):
        plan(2, nb.OCC_NONE, [(7, X, Y, 0, 0, 0)])
    with pytest.raises(nb.NbError):
        plan(2, nb.OCC_NONE, [(nb.SK_DOT, X, Y, 0, 0, 5000)])
    with pytest.raises(nb.NbError):
        plan(0, nb.OCC_NONE)


def test_listing3_cg_plan_structure():
    """Listing 3 CG (L154-L163) with device scalars: the halo of p precedes
    the stencil; alpha waits for <p, q> and feeds both updates; beta waits
    for <r, r>; under Two-way OCC the UpdateP map and the stencil split and
    the internal stencil is hinted before the halo (Fig. 4d pattern)."""
    P_, Q_, R_, X_ = 0, 1, 2, 3
    RR, PQ, AL, BE, RR2 = 0, 1, 2, 3, 4
    C = [(nb.SK_AXPBY, R_, P_, 1.0, 1.0, 0, -1, BE, 0),
         (nb.SK_POISSON, P_, Q_, 0.0, 0.0, 0),
         (nb.SK_DOT, P_, Q_, 0.0, 0.0, PQ),
         (nb.SK_SCALAR, RR, PQ, 0.0, 0.0, AL, -1, -1, nb.SC_DIV),
         (nb.SK_AXPBY, P_, X_, 1.0, 1.0, 0, AL, -1, 0),
         (nb.SK_AXPBY, Q_, R_, -1.0, 1.0, 0, AL, -1, 0),
         (nb.SK_DOT, R_, R_, 0.0, 0.0, RR2),
         (nb.SK_SCALAR, RR2, RR, 0.0, 0.0, BE, -1, -1, nb.SC_DIV),
         (nb.SK_SCALAR, RR2, 0, 0.0, 0.0, RR, -1, -1, nb.SC_COPY)]
    plan = nb.nb_skeleton_plan(4, nb.OCC_TWO_WAY, C)
    nodes = plan["nodes"]
    names = [n["name"] for n in nodes]
    edges = set(map(tuple, plan["data"]))
    idx = {nm: i for i, nm in enumerate(names)}

    def path(a, b):
        adj = {}
        for u, v in edges:
            adj.setdefault(u, []).append(v)
        st, seen = [a], set()
        while st:
            u = st.pop()
            if u == b:
                return True
            for v in adj.get(u, []):
                if v not in seen:
                    seen.add(v)
                    st.append(v)
        return False
    assert "halo(f0)" in names
    assert "axpby#0[bnd]" in names and "axpby#0[int]" in names       # UpdateP split (Extended)
    assert "poisson#1[int]" in names and "poisson#1[bnd]" in names
    assert path(idx["halo(f0)"], idx["poisson#1[bnd]"])
    assert not path(idx["halo(f0)"], idx["poisson#1[int]"])           # internal stencil overlaps the halo
    assert (idx["poisson#1[int]"], idx["halo(f0)"]) in set(map(tuple, plan["hints"]))
    # alpha after <p, q>; both updates after alpha; beta after <r, r>; rr copy after beta (WaR on rr)
    dot_pq = [i for i, nm in enumerate(names) if nm.startswith("dot#2") and nodes[i]["finalize"]][0]
    assert path(dot_pq, idx["scalar#3"])
    def parts_of(prefix):
        return [i for i, nm in enumerate(names) if nm.split("[")[0] == prefix]
    for u in parts_of("axpby#4") + parts_of("axpby#5"):  # r <- r - alpha q consumes q: split (Two-way)
        assert path(idx["scalar#3"], u)
    assert len(parts_of("axpby#5")) == 2
    dot_rr = [i for i, nm in enumerate(names) if nm.startswith("dot#6") and nodes[i]["finalize"]][0]
    assert path(dot_rr, idx["scalar#7"]) and path(idx["scalar#7"], idx["scalar#8"])
    # the x and r updates touch disjoint data: concurrent
    for u in parts_of("axpby#4"):
        for v in parts_of("axpby#5"):
            assert not path(u, v) and not path(v, u)
    assert plan["streams"] >= 2
