"""Oracle (TEST INFRASTRUCTURE ONLY — never imported by the product path):
one training step of the IP emulator.

PAPER.md §3.1, molecular-design steps (3) "use the data from the
previous steps to train an ML model that acts as an emulator of the
simulations" and (7) "train a new emulator"; §3.4: training and
inference are the workflow's GPU phases. The paper gives no loss, optimiser
or schedule; the readings (R10) are:
  * loss  L = (1/M) sum_m (y_m - t_m)^2 over the task's M molecules (targets t
    are task inputs: the "computed IPs" of step (2));
  * one plain SGD step  theta <- theta - lr * dL/dtheta  on every parameter
    (E_atom, W_b, U, c, W1, c1, w2, c2), lr a task input;
  * parameters are fp32 training state initialised from the seeded bf16-exact
    values of C1 (the same numbers as the inference function).
The forward pass is C4 (oracle/mpnn.py) with its intermediate values kept;
the backward pass is the chain rule written out step by step in reverse
order (no autograd), float64 throughout:
  readout   r = sum_v h_v^T, a = W1 r + c1, z = ReLU(a), y = w2.z + c2
            dy = 2 (y - t) / M ; dw2 += dy z ; dc2 += dy ; da = dy w2 * [a > 0]
            dW1 += da r^T ; dc1 += da ; dh^T_v = W1^T da  (every atom v of m)
  step t    h^{t+1} = ReLU(q),  q_v = U h^t_v + sum_{(u,b) in N(v)} W_b h^t_u + c
            dq = dh^{t+1} * [h^{t+1} > 0] ; dU += dq_v h_v^T ; dc += dq_v
            dW_b += dq_v h_u^T for every (u, b) in N(v)
            dh^t_v = U^T dq_v + sum_{(u,b) in N(v)} W_b^T dq_u
  embedding dE[a_v] += dh^0_v
Pinned by tests/test_oracle_mpnn_train.py: central finite differences of the
loss for every tensor, an independent torch.autograd fp64 formulation, lr = 0
invariance and the loss of the inference oracle's outputs.
"""
from __future__ import annotations

import numpy as np

from oracle.mpnn import relu

PARAMS = ("e_atom", "w_b", "u", "c", "w1", "c1", "w2", "c2")


def as_f64(w: dict) -> dict:
    return {k: np.array(w[k], dtype=np.float64) for k in PARAMS}


def _neighbours(n, edges):
    """N(v) = [(u, b)] in edge order (each bond contributes to both ends)."""
    nb = [[] for _ in range(n)]
    for (u, v, b) in edges:
        nb[v].append((u, b))
        nb[u].append((v, b))
    return nb


def molecule_grad(w: dict, types, edges, steps: int, target: float, M: int):
    """Forward + backward of one molecule's loss term (1/M)(y - t)^2.
    Returns (y, grads dict)."""
    E, Wb, U, c = w["e_atom"], w["w_b"], w["u"], w["c"]
    W1, c1, w2, c2 = w["w1"], w["c1"], w["w2"], float(w["c2"])
    types = np.asarray(types, dtype=np.int64)
    n = len(types)
    nb = _neighbours(n, edges)
    hs = [E[types].copy()]
    for _ in range(steps):
        h = hs[-1]
        q = h @ U.T + c
        for v in range(n):
            for (u, b) in nb[v]:
                q[v] += Wb[b] @ h[u]
        hs.append(relu(q))
    r = hs[-1].sum(axis=0)
    a = W1 @ r + c1
    z = relu(a)
    y = float(w2 @ z + c2)
    g = {k: np.zeros_like(np.asarray(w[k], dtype=np.float64)) for k in PARAMS}
    dy = 2.0 * (y - target) / M
    g["w2"] += dy * z
    g["c2"] += dy
    da = dy * w2 * (a > 0)
    g["w1"] += np.outer(da, r)
    g["c1"] += da
    dh = np.tile(W1.T @ da, (n, 1))
    for t in range(steps - 1, -1, -1):
        h, hn = hs[t], hs[t + 1]
        dq = dh * (hn > 0)
        g["u"] += dq.T @ h
        g["c"] += dq.sum(axis=0)
        dh_new = dq @ U
        for v in range(n):
            for (u, b) in nb[v]:
                g["w_b"][b] += np.outer(dq[v], h[u])
                dh_new[u] += Wb[b].T @ dq[v]
        dh = dh_new
    for v in range(n):
        g["e_atom"][types[v]] += dh[v]
    return y, g


def train_step(w: dict, task: dict, targets, steps: int, lr: float):
    """One SGD step over all molecules of a CSR task dict. Returns
    (new params float64, loss, y[M] predictions before the update)."""
    from workloads.inputs import molecule_of
    w = as_f64(w)
    M = len(task["atom_off"]) - 1
    grads = {k: np.zeros_like(w[k]) for k in PARAMS}
    ys = np.empty(M)
    for m in range(M):
        types, edges = molecule_of(task, m)
        ys[m], g = molecule_grad(w, types, edges, steps, float(targets[m]), M)
        for k in PARAMS:
            grads[k] += g[k]
    loss = float(np.mean((ys - np.asarray(targets, dtype=np.float64)) ** 2))
    new = {k: w[k] - lr * grads[k] for k in PARAMS}
    return new, loss, ys, grads


def loss_only(w: dict, task: dict, targets, steps: int) -> float:
    """L(theta) through the inference oracle (for finite differences)."""
    from oracle.mpnn import mpnn_task
    y = mpnn_task(w, task, steps)
    return float(np.mean((y - np.asarray(targets, dtype=np.float64)) ** 2))
