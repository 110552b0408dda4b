"""Pins for the MPNN (IP-emulator) oracle. The architecture is reading A22
(§3.1 P:109 names the emulator but not its model): parity vs the paper
is unpinned; these tests pin the oracle to mathematics instead."""
import numpy as np

from oracle import mpnn as om
from workloads.configs import MPNN
from workloads.inputs import molecules, molecule_of
from workloads.weights import mpnn_weights

W = mpnn_weights(MPNN)
T = MPNN.steps


def _dense_y(w, types, edges, steps):
    """Independent dense reformulation in float64: m = sum_b A_b H W_b^T with
    symmetric per-type adjacency A_b (built here, not from the oracle)."""
    n = len(types)
    A = np.zeros((4, n, n))
    for u, v, b in edges:
        A[b, u, v] += 1.0
        A[b, v, u] += 1.0
    H = np.asarray(w["e_atom"], np.float64)[types]
    for _ in range(steps):
        M = sum(A[b] @ H @ np.asarray(w["w_b"][b], np.float64).T for b in range(4))
        H = np.maximum(H @ np.asarray(w["u"], np.float64).T + M + w["c"], 0)
    r = H.sum(0)
    z = np.maximum(np.asarray(w["w1"], np.float64) @ r + w["c1"], 0)
    return float(np.asarray(w["w2"], np.float64) @ z + float(w["c2"]))


def test_mpnn_matches_dense_reformulation():
    task = molecules(3, 12)
    for m in range(12):
        types, edges = molecule_of(task, m)
        a = om.mpnn_molecule(W, types, edges, T)
        b = _dense_y(W, types, edges, T)
        assert abs(a - b) <= 1e-12 * max(1.0, abs(b))


def test_mpnn_single_atom_no_bonds_closed_form():
    # no bonds: m = 0, so h_T = (ReLU o (U . + c))^T applied to E_atom[a]; checked by
    # unrolling with torch (independent library) in float64.
    import torch
    for a in range(8):
        h = torch.tensor(np.asarray(W["e_atom"][a], np.float64))
        U = torch.tensor(np.asarray(W["u"], np.float64))
        c = torch.tensor(np.asarray(W["c"], np.float64))
        for _ in range(T):
            h = torch.relu(torch.mv(U, h) + c)
        z = torch.relu(torch.mv(torch.tensor(np.asarray(W["w1"], np.float64)), h)
                       + torch.tensor(np.asarray(W["c1"], np.float64)))
        y = float(torch.dot(torch.tensor(np.asarray(W["w2"], np.float64)), z)) + float(W["c2"])
        assert abs(om.mpnn_molecule(W, [a], [], T) - y) < 1e-12


def test_mpnn_permutation_invariance_and_bond_direction():
    task = molecules(5, 4)
    rng = np.random.default_rng(0)
    for m in range(4):
        types, edges = molecule_of(task, m)
        n = len(types)
        perm = rng.permutation(n)            # new label of old atom i = perm[i]
        t2 = [0] * n
        for i in range(n):
            t2[perm[i]] = types[i]
        e2 = [(int(perm[v]), int(perm[u]), b) for u, v, b in edges]   # relabel + flip direction
        y1 = om.mpnn_molecule(W, types, edges, T)
        y2 = om.mpnn_molecule(W, t2, e2, T)
        assert abs(y1 - y2) <= 1e-10 * max(1, abs(y1))


def test_mpnn_readout_additivity_disjoint_union():
    # r(G1 u G2) = r(G1) + r(G2): with w2 = e_k, c1 = 0, W1 = I and c2 = 0 the output is
    # ReLU(r)_k; choose k where both r are >= 0 so y(union) = y(G1) + y(G2).
    task = molecules(9, 2)
    g1, g2 = molecule_of(task, 0), molecule_of(task, 1)
    n1 = len(g1[0])
    union_t = g1[0] + g2[0]
    union_e = g1[1] + [(u + n1, v + n1, b) for u, v, b in g2[1]]
    w = dict(W)
    w["w1"] = np.eye(128)
    w["c1"] = np.zeros(128)
    w["c2"] = 0.0
    hits = 0
    for k in range(128):
        w["w2"] = np.eye(128)[k]
        y1 = om.mpnn_molecule(w, *g1, T)
        y2 = om.mpnn_molecule(w, *g2, T)
        if y1 > 0 and y2 > 0:
            yu = om.mpnn_molecule(w, union_t, union_e, T)
            assert abs(yu - (y1 + y2)) <= 1e-12 * max(1, abs(yu))
            hits += 1
            if hits >= 3:
                break
    assert hits >= 1


def test_mpnn_outputs_finite_and_vary():
    task = molecules(1, 16)
    y = om.mpnn_task(W, task, T)
    assert np.all(np.isfinite(y)) and np.std(y) > 0
