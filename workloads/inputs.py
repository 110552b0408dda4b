"""Seeded synthetic inputs: prompts, molecular graphs, task-mix order.

SURVEY.md §8(c) C1 is the recipe. Only integer generation lives here (no
arithmetic of the method). Shared by the oracle tests and the harness; the
CUDA library receives the results through `fn_submit`.
"""
from __future__ import annotations

import numpy as np

from .prng import draw, draw_int, key

BOND_DTYPE = np.dtype([("u", "<i2"), ("v", "<i2"), ("bond", "u1"), ("pad", "u1")])
assert BOND_DTYPE.itemsize == 6


# ---------------------------------------------------------------------------
# Prompts (C1): token j of sequence b of task k = draw(key(seed_p, k*256 + b), j) mod V
# k is the 1-based task id inside its workload.
# ---------------------------------------------------------------------------

def prompt_tokens(task_id: int, batch: int, prompt_len: int, vocab: int,
                  seed: int = 0xC0FFEE) -> np.ndarray:
    out = np.empty((batch, prompt_len), dtype=np.int32)
    for b in range(batch):
        k = np.uint64(key(seed, task_id * 256 + b))
        r = draw(k, np.arange(prompt_len, dtype=np.uint64))
        out[b] = (r % np.uint64(vocab)).astype(np.int32)
    return out


def ip_targets(task_id: int, n_mol: int, seed: int = 0x1B7) -> np.ndarray:
    """Synthetic training targets ("computed IPs", §3.1 P:109 step (2))
    for the N4 training step: t_m = ((draw(key(seed, task_id), m) >> 40) / 2^24)
    * 2 - 1, uniform in [-1, 1), exactly representable in fp32."""
    r = draw(np.uint64(key(seed, task_id)), np.arange(n_mol, dtype=np.uint64))
    return ((r >> np.uint64(40)).astype(np.float64) / float(1 << 24) * 2.0 - 1.0).astype(np.float32)


# ---------------------------------------------------------------------------
# Molecules (C1): molecule j of task k uses a sequential counter i over
# draw(key(seed_g, k*2^20 + j), i):
#   n = 10 + r mod 21 ; n atom types r mod 8 ;
#   for v = 1..n-1: parent = r mod v, bond = r mod 4   (tree edge (parent, v))
#   kc = r mod 3 ring closures, each 3 draws u = r mod n, w = r mod n, b = r mod 4,
#   accepted iff u != w and {u, w} not already bonded (draws consumed regardless).
# ---------------------------------------------------------------------------

def molecule_slow(task_id: int, j: int, seed: int = 0x6A5):
    """Plain scalar generator (the readable definition). Returns (types, edges)."""
    s = key(seed, task_id * (1 << 20) + j)
    i = 0

    def r():
        nonlocal i
        v = draw_int(s, i)
        i += 1
        return v

    n = 10 + r() % 21
    types = [r() % 8 for _ in range(n)]
    edges = []
    bonded = set()
    for v in range(1, n):
        parent = r() % v
        bond = r() % 4
        edges.append((parent, v, bond))
        bonded.add((min(parent, v), max(parent, v)))
    kc = r() % 3
    for _ in range(kc):
        u = r() % n
        w = r() % n
        b = r() % 4
        if u != w and (min(u, w), max(u, w)) not in bonded:
            edges.append((u, w, b))
            bonded.add((min(u, w), max(u, w)))
    return types, edges


def molecules(task_id: int, n_mol: int, seed: int = 0x6A5):
    """Vectorised generator for a task of n_mol molecules, CSR layout.

    Returns dict(atom_off[int32, M+1], atom_type[uint8], edge_off[int32, M+1],
    edges[BOND_DTYPE]). Identical to `molecule_slow` (pinned by a test).
    """
    M = n_mol
    keys = np.array([key(seed, task_id * (1 << 20) + j) for j in range(M)], dtype=np.uint64)
    kcol = keys[:, None]
    n = (10 + draw(keys, 0) % np.uint64(21)).astype(np.int64)            # [M]
    # atom types at i = 1..n
    ti = np.arange(1, 31, dtype=np.uint64)[None, :]
    types_all = (draw(kcol, ti) % np.uint64(8)).astype(np.uint8)          # [M, 30]
    # tree edges: v = 1..n-1 at i = 1 + n + 2(v-1), +1
    v = np.arange(1, 30, dtype=np.int64)[None, :]                         # [1, 29]
    base = (1 + n)[:, None] + 2 * (v - 1)                                 # [M, 29]
    rp = draw(kcol, base.astype(np.uint64))
    rb = draw(kcol, (base + 1).astype(np.uint64))
    parent = (rp % v.astype(np.uint64)).astype(np.int64)
    bond = (rb % np.uint64(4)).astype(np.int64)
    # ring closures: kc at i = 3n - 1, closure c at 3n + 3c + {0,1,2}
    ikc = 3 * n - 1
    kc = (draw(keys, ikc.astype(np.uint64)) % np.uint64(3)).astype(np.int64)
    c = np.arange(2, dtype=np.int64)[None, :]
    cb = (3 * n)[:, None] + 3 * c
    nu = n.astype(np.uint64)[:, None]
    cu = (draw(kcol, cb.astype(np.uint64)) % nu).astype(np.int64)
    cw = (draw(kcol, (cb + 1).astype(np.uint64)) % nu).astype(np.int64)
    cbond = (draw(kcol, (cb + 2).astype(np.uint64)) % np.uint64(4)).astype(np.int64)

    atom_off = np.zeros(M + 1, dtype=np.int32)
    atom_off[1:] = np.cumsum(n)
    atom_type = np.concatenate([types_all[m, :n[m]] for m in range(M)]).astype(np.uint8)
    edge_lists = []
    for m in range(M):
        nm = int(n[m])
        e_u = parent[m, :nm - 1]
        e_v = np.arange(1, nm)
        e_b = bond[m, :nm - 1]
        rows = [np.stack([e_u, e_v, e_b], axis=1)]
        bonded = set(zip(np.minimum(e_u, e_v).tolist(), np.maximum(e_u, e_v).tolist()))
        for q in range(int(kc[m])):
            u, w, b = int(cu[m, q]), int(cw[m, q]), int(cbond[m, q])
            pr = (min(u, w), max(u, w))
            if u != w and pr not in bonded:
                rows.append(np.array([[u, w, b]], dtype=np.int64))
                bonded.add(pr)
        edge_lists.append(np.concatenate(rows, axis=0))
    ne = np.array([len(e) for e in edge_lists], dtype=np.int64)
    edge_off = np.zeros(M + 1, dtype=np.int32)
    edge_off[1:] = np.cumsum(ne)
    allE = np.concatenate(edge_lists, axis=0)
    edges = np.zeros(len(allE), dtype=BOND_DTYPE)
    edges["u"] = allE[:, 0]
    edges["v"] = allE[:, 1]
    edges["bond"] = allE[:, 2]
    return dict(atom_off=atom_off, atom_type=atom_type, edge_off=edge_off, edges=edges)


def molecule_of(task: dict, m: int):
    """Slice molecule m out of a CSR task dict -> (types[int], edges[(u,v,b)])."""
    a0, a1 = int(task["atom_off"][m]), int(task["atom_off"][m + 1])
    e0, e1 = int(task["edge_off"][m]), int(task["edge_off"][m + 1])
    e = task["edges"][e0:e1]
    return (task["atom_type"][a0:a1].astype(int).tolist(),
            list(zip(e["u"].astype(int).tolist(), e["v"].astype(int).tolist(),
                     e["bond"].astype(int).tolist())))


# ---------------------------------------------------------------------------
# Task-mix shuffle (C1): Fisher-Yates with j = draw(key(42, 0), n-1-i) mod (i+1)
# ---------------------------------------------------------------------------

def shuffle(items: list, seed: int = 42) -> list:
    items = list(items)
    n = len(items)
    k = key(seed, 0)
    for i in range(n - 1, 0, -1):
        j = draw_int(k, n - 1 - i) % (i + 1)
        items[i], items[j] = items[j], items[i]
    return items
