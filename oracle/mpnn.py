"""Oracle: the scientific-computing function — IP-emulator inference.

PAPER.md §3.1, molecular-design step (4): "use the trained emulator to
estimate the IPs of a larger pool of newly generated molecules"; §3.4
training and inference are the GPU phases. The paper does not specify the
emulator (ambiguity register A22); the message-passing network below is the
reading SURVEY.md §8(c) C4 adopts. PARITY VS THE PAPER IS UNPINNED for this
function (no architecture or numbers in the paper); oracle-vs-GPU parity and
the oracle's own mathematical pins (closed forms, invariants, an independent
dense reformulation) are what is checked.

    h_v = E_atom[a_v]
    repeat T times (simultaneous update):
        m_v = sum over bonds (u,v,b) or (v,u,b) of W_b h_u
        h_v = ReLU(U h_v + m_v + c)
    r = sum_v h_v ;  y = w2 . ReLU(W1 r + c1) + c2
"""
from __future__ import annotations

import numpy as np


def relu(z):
    return np.maximum(z, 0.0)


def mpnn_molecule(w: dict, types, edges, steps: int) -> float:
    """Literal C4 for one molecule. types[n] ints, edges [(u, v, b)]."""
    f64 = lambda a: np.asarray(a, dtype=np.float64)
    E, Wb, U, c = f64(w["e_atom"]), f64(w["w_b"]), f64(w["u"]), f64(w["c"])
    h = E[np.asarray(types, dtype=np.int64)].copy()
    for _ in range(steps):
        m = np.zeros_like(h)
        for (u, v, b) in edges:
            m[v] += Wb[b] @ h[u]
            m[u] += Wb[b] @ h[v]
        h = relu(h @ U.T + m + c)
    r = h.sum(axis=0)
    return float(f64(w["w2"]) @ relu(f64(w["w1"]) @ r + f64(w["c1"])) + float(w["c2"]))


def mpnn_task(w: dict, task: dict, steps: int) -> np.ndarray:
    """All molecules of a CSR task dict (workloads.inputs.molecules) -> y[M] float64."""
    from workloads.inputs import molecule_of
    M = len(task["atom_off"]) - 1
    out = np.empty(M)
    for m in range(M):
        types, edges = molecule_of(task, m)
        out[m] = mpnn_molecule(w, types, edges, steps)
    return out
