"""Pins of the N4 training-step oracle (oracle/mpnn_train.py) against things
other than itself: central finite differences of the loss, an independent
torch.autograd formulation in float64 (dense adjacency, library backprop),
the inference oracle (lr = 0) and first-order descent."""
import numpy as np
import torch

from oracle import mpnn as om
from oracle import mpnn_train as ot
from workloads.configs import MPNN
from workloads.inputs import molecules, ip_targets, molecule_of
from workloads.weights import mpnn_weights


def _random_weights(F, seed=7, n_types=8, n_bonds=4):
    rng = np.random.default_rng(seed)
    g = lambda *s: rng.normal(0.0, 0.35, size=s)
    return dict(e_atom=g(n_types, F), w_b=g(n_bonds, F, F), u=g(F, F), c=g(F), w1=g(F, F),
                c1=g(F), w2=g(F), c2=np.float64(rng.normal()))


def test_gradients_match_central_finite_differences():
    F = 6
    w = _random_weights(F)
    task = molecules(3, 2)
    t = ip_targets(3, 2).astype(np.float64)
    _, loss, _, grads = ot.train_step(w, task, t, MPNN.steps, lr=0.0)
    assert abs(loss - ot.loss_only(w, task, t, MPNN.steps)) < 1e-12 * max(1.0, loss)
    eps = 1e-6
    for k in ot.PARAMS:
        base = np.array(w[k], dtype=np.float64)
        flat = base.reshape(-1)
        for i in range(flat.size):
            wp = dict(w)
            wm = dict(w)
            xp, xm = flat.copy(), flat.copy()
            xp[i] += eps
            xm[i] -= eps
            wp[k] = xp.reshape(base.shape)
            wm[k] = xm.reshape(base.shape)
            fd = (ot.loss_only(wp, task, t, MPNN.steps) - ot.loss_only(wm, task, t, MPNN.steps)) / (2 * eps)
            an = np.asarray(grads[k]).reshape(-1)[i]
            assert abs(fd - an) <= 1e-6 * max(1.0, abs(fd)), (k, i, fd, an)


def _torch_loss(w, task, targets, steps):
    """Independent formulation: dense per-type adjacency A_b, m = sum_b A_b H W_b^T,
    torch autograd for the backward pass."""
    P = {k: torch.tensor(np.asarray(w[k], dtype=np.float64), requires_grad=True) for k in ot.PARAMS}
    M = len(task["atom_off"]) - 1
    ys = []
    for m in range(M):
        types, edges = molecule_of(task, m)
        n = len(types)
        A = torch.zeros(4, n, n, dtype=torch.float64)
        for (u, v, b) in edges:
            A[b, v, u] += 1.0
            A[b, u, v] += 1.0
        h = P["e_atom"][torch.tensor(np.asarray(types, dtype=np.int64))]
        for _ in range(steps):
            msg = sum(A[b] @ h @ P["w_b"][b].T for b in range(P["w_b"].shape[0]))
            h = torch.relu(h @ P["u"].T + msg + P["c"])
        r = h.sum(0)
        ys.append(P["w2"] @ torch.relu(P["w1"] @ r + P["c1"]) + P["c2"])
    y = torch.stack(ys)
    loss = ((y - torch.tensor(np.asarray(targets, dtype=np.float64))) ** 2).mean()
    loss.backward()
    return float(loss.detach()), {k: P[k].grad.numpy() for k in ot.PARAMS}, y.detach().numpy()


def test_gradients_match_torch_autograd_full_width():
    w = mpnn_weights(MPNN)
    task = molecules(5, 3)
    t = ip_targets(5, 3)
    _, loss, ys, grads = ot.train_step(w, task, t, MPNN.steps, lr=0.0)
    tl, tg, ty = _torch_loss(w, task, t, MPNN.steps)
    assert abs(loss - tl) <= 1e-12 * max(1.0, abs(tl))
    assert np.allclose(ys, ty, rtol=1e-12, atol=1e-12)
    for k in ot.PARAMS:
        ref = np.asarray(tg[k])
        scale = max(1e-30, float(np.max(np.abs(ref))))
        assert np.max(np.abs(np.asarray(grads[k]) - ref)) <= 1e-10 * scale, k


def test_lr_zero_is_identity_and_predictions_match_inference_oracle():
    w = mpnn_weights(MPNN)
    task = molecules(9, 4)
    t = ip_targets(9, 4)
    new, loss, ys, _ = ot.train_step(w, task, t, MPNN.steps, lr=0.0)
    for k in ot.PARAMS:
        assert np.array_equal(new[k], np.asarray(w[k], dtype=np.float64))
    assert np.allclose(ys, om.mpnn_task(w, task, MPNN.steps), rtol=1e-13, atol=1e-13)
    assert loss == float(np.mean((ys - t.astype(np.float64)) ** 2))


def test_small_sgd_step_decreases_loss():
    w = _random_weights(8, seed=11)
    task = molecules(4, 3)
    t = ip_targets(4, 3)
    lr = 1e-4
    new, loss, _, grads = ot.train_step(w, task, t, MPNN.steps, lr=lr)
    after = ot.loss_only(new, task, t, MPNN.steps)
    gn = sum(float(np.sum(np.asarray(g) ** 2)) for g in grads.values())
    assert after < loss
    # first order: L(theta - lr g) ~ L - lr |g|^2
    assert abs((loss - after) - lr * gn) <= 0.05 * lr * gn


def test_targets_generator_range_and_determinism():
    t = ip_targets(1, 1000)
    assert t.dtype == np.float32 and np.all(t >= -1) and np.all(t < 1)
    assert np.array_equal(t, ip_targets(1, 1000))
    assert not np.array_equal(t, ip_targets(2, 1000))
