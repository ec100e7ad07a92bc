"""Pins of the seeded input generators (synth/), independent of the oracle and the CUDA path.

* 2D triple point IE_0 = 10.05 = Table 6's total energy, exact in rationals
* 3D triple point (C5, zone-centre material rule) IE_0 = 19509/640 = 30.4828125
* Sedov: sum IE = E_b = 0.25
IE = sum_z rho0|J0| sum_j E_zj / k^d (each Bernstein function integrates to 1/k^d on [0,1]^d).
"""
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import synth


def internal_energy(mesh, st):
    return float((st.e.sum(1) * st.rho0detJ0[:, 0]).sum() / mesh.nt)


def test_triple_point_2d_table6():
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_values.json")))
    m = synth.triple_point_mesh(2, 3, (56, 24))
    s = synth.triple_point_s0(m)
    ie = internal_energy(m, s)
    target = gold["table6_triple_point_total_energy"]["value"]
    assert abs(ie - target) < 1e-12
    # exact: left 1x3 at p=1, two 6x1.5 right regions at p=0.1 with gamma 1.5 / 1.4
    exact = Fraction(1) / Fraction(1, 2) * 3 + Fraction(1, 10) / Fraction(1, 2) * 9 + Fraction(1, 10) / Fraction(2, 5) * 9
    assert exact == Fraction(201, 20)


def test_triple_point_3d_c5_energy():
    m = synth.triple_point_mesh(3, 1, (48, 24, 24))   # order does not change IE
    s = synth.triple_point_s0(m)
    assert abs(internal_energy(m, s) - 19509 / 640) < 1e-11
    assert sorted(np.unique(m.zone_mat).tolist()) == [0, 1, 2]


@pytest.mark.parametrize("name", ["C1", "C2", "C3"])
def test_sedov_energy(name):
    m, s = synth.config(name, "S0")
    assert abs(internal_energy(m, s) - 0.25) < 1e-15


def test_mesh_numbering():
    m = synth.box_mesh(3, 2, (2, 3, 4))
    assert m.num_nodes == 5 * 7 * 9
    assert m.zone_nodes.shape == (24, 27)
    # zone 0 local node 0 is the origin, last local node of the last zone is the far corner
    assert np.all(m.x0[:, m.zone_nodes[0, 0]] == 0)
    assert np.allclose(m.x0[:, m.zone_nodes[-1, -1]], 1.0)
    # x-fastest local ordering: local node 1 differs from node 0 only in x
    d = m.x0[:, m.zone_nodes[:, 1]] - m.x0[:, m.zone_nodes[:, 0]]
    assert np.all(d[0] > 0) and np.all(d[1:] == 0)
    # every node is used
    assert np.unique(m.zone_nodes).size == m.num_nodes


def test_seeded_reproducible():
    a = synth.config("C1", "S1")[1]
    b = synth.config("C1", "S1")[1]
    c = synth.config("C1", "S1b")[1]
    assert np.array_equal(a.x, b.x) and np.array_equal(a.e, b.e)
    assert not np.array_equal(a.v, c.v)


def test_s1_boundary_fixed():
    m, s = synth.config("C3", "S1", N=(4, 4, 4))
    onb = np.zeros(m.num_nodes, bool)
    for t in range(3):
        onb |= (m.x0[t] == 0) | (m.x0[t] == 1)
    assert np.abs(s.x[:, onb] - m.x0[:, onb]).max() < 1e-15


@pytest.mark.parametrize("dim,P", [(2, 2), (2, 4), (2, 8), (3, 2), (3, 4), (3, 8)])
def test_partition(dim, P):
    N = (8, 6) if dim == 2 else (4, 4, 6)
    m = synth.box_mesh(dim, 2, N)
    parts = synth.partition(m, P)
    allz = np.concatenate([p.zones for p in parts])
    assert np.array_equal(np.sort(allz), np.arange(m.num_zones))
    owners = np.zeros(m.num_nodes, int)
    for p in parts:
        assert np.array_equal(p.nodes[p.zone_nodes], m.zone_nodes[p.zones])
        owners[p.nodes[p.owned]] += 1
        for i, q in enumerate(p.nbr_rank):
            loc = p.nbr_nodes[p.nbr_offset[i]:p.nbr_offset[i + 1]]
            g = p.nodes[loc]
            assert np.all(np.diff(g) > 0)
            other = parts[q]
            assert np.array_equal(np.intersect1d(p.nodes, other.nodes), g)
    assert np.all(owners == 1)   # owner rule: every node counted exactly once


@pytest.mark.parametrize("name,N,k,P", [("C4", (8, 6, 4), 2, 8), ("C3", (6, 6, 6), None, 4), ("C2", (10, 8), 3, 8),
                                        ("C2", (6, 4), 2, 2)])
def test_partition_numbers_boundary_zones_first(name, N, k, P):
    """synth.partition numbers each rank's zones boundary-first (the zones touching a node shared with another
    rank, then the interior ones, each group ascending): the numbering the library's overlap schedule needs
    (blast_cf_exchange_schedule); every zone appears on exactly one rank."""
    m, _ = synth.config(name, "S1", N=N, k=k)
    parts = synth.partition(m, P)
    seen = np.concatenate([p.zones for p in parts])
    assert np.array_equal(np.sort(seen), np.arange(m.num_zones))
    for p in parts:
        shared = np.zeros(len(p.nodes), dtype=bool)
        shared[p.nbr_nodes] = True
        bnd = shared[p.zone_nodes].any(axis=1)
        nb = int(bnd.sum())
        assert bnd[:nb].all() and not bnd[nb:].any()
        assert np.all(np.diff(p.zones[:nb]) > 0) and np.all(np.diff(p.zones[nb:]) > 0)
        # every rank of a 2 x ... x 2 block partition shares a node with every other (dt piggy-back)
        if max(synth.block_dims(m.dim, P)) <= 2:
            assert len(p.nbr_rank) == P - 1
