"""D5 task farm driver (SURVEY.md §8(d) D5, configs[4]): a closed stream of
mixed tasks (50/50 GPT-2s decode / 1024-molecule MPNN, shuffled with seed 42)
placed by WLAW over 7 fill partitions, with the layout alternating between
fill-7 and LAYOUT_B via part_resize between waves of submissions (§6
P:242, §7: re-partitioning without a restart).

Used by tools/suite.py c5 (measurement) and tests/test_gpu_farm_d5.py (the
D5 correctness checks: trace vs the simulator, invariants, sampled oracle
parity). This module drives the C ABI only; every call that changes the
canonical trace is appended to `events` so a checker can replay it.
"""
from __future__ import annotations

import time

from workloads.configs import GPT2S, MPNN, LAYOUTS_FILL
from workloads.inputs import molecules, prompt_tokens, shuffle

P_LEN, G_LEN = 16, 32
MOLS = 1024
LAYOUT_B = [40, 40, 16, 16, 16, 8, 8]


class Farm:
    def __init__(self, mx, mol_variants: int = 16, quota: int = 1 << 30):
        self.mx = mx
        self.quota = quota
        self.events = []          # ("create", gpu, sm, hbm) / ("resize", part, sm, hbm) /
        #                           ("destroy", part) / ("submit", fn, part, cost)
        self.fd_desc = mx.decode_desc(GPT2S)
        self.fm_desc = mx.mpnn_desc(MPNN, MOLS, MOLS * 30, MOLS * 32)
        self.fd = mx.fn_register(self.fd_desc)
        self.fm = mx.fn_register(self.fm_desc)
        self.mol_cache = [molecules(k, MOLS) for k in range(1, mol_variants + 1)]
        self.cost_d = None

    # --- trace-recorded wrappers ------------------------------------------------
    def create(self, gpu, sm):
        p = self.mx.part_create(gpu, sm, self.quota)
        self.events.append(("create", gpu, sm, self.quota))
        return p

    def resize(self, part, sm):
        self.mx.part_resize(part, sm, 0)
        self.events.append(("resize", part, sm, 0))

    def destroy(self, part):
        self.mx.part_destroy(part)
        self.events.append(("destroy", part))

    def submit(self, part, kind, task):
        desc = self.fd_desc if kind == "d" else self.fm_desc
        if kind == "d" and self.cost_d is not None:
            cost = self.cost_d
        else:
            cost = self.mx.task_default_cost(desc, task)
            if kind == "d":
                self.cost_d = cost
        self.mx.fn_submit(part, task)
        self.events.append(("submit", self.fd if kind == "d" else self.fm, part, cost))

    # --- workload ---------------------------------------------------------------
    def items(self, n_dec, n_mpnn):
        """[(kind, k, Task)]: decode task k uses prompt_tokens(k, ...), MPNN task k
        the molecule set mol_cache[(k-1) % variants]."""
        kinds = shuffle([("d", k) for k in range(1, n_dec + 1)] +
                        [("m", k) for k in range(1, n_mpnn + 1)], 42)
        out = []
        for kind, k in kinds:
            if kind == "d":
                out.append(("d", k, self.mx.decode_task(
                    self.fd, prompt_tokens(k, 1, P_LEN, GPT2S.vocab), G_LEN)))
            else:
                out.append(("m", k, self.mx.mpnn_task(self.fm, self.mol_of(k))))
        return out

    def mol_of(self, k):
        return self.mol_cache[(k - 1) % len(self.mol_cache)]

    def apply_layout(self, parts, sizes):
        """Resize partitions to `sizes` (shrinks first so growing ones find free groups)."""
        cur = [self.mx.part_query(p)["sm_count"] for p in parts]
        order = sorted(range(len(parts)), key=lambda i: sizes[i] - cur[i])
        lat_ms = []
        for i in order:
            if sizes[i] != cur[i]:
                h0 = time.perf_counter()
                self.resize(parts[i], sizes[i])
                lat_ms.append((time.perf_counter() - h0) * 1e3)
        return lat_ms

    def run(self, sizes, n_tasks, resize_every=0, warm=True):
        """One farm run on partitions of `sizes` (GPU 0). Waves of `resize_every`
        submissions; before wave w >= 2 is submitted, wave w-2 is collected and
        (if resize_every) the layout flips fill-7 <-> LAYOUT_B, so every resize
        happens while about one wave of work is queued or running. Returns
        dict(items, results, resize_ms, wall_s, parts_info)."""
        mx = self.mx
        parts = [self.create(0, s) for s in sizes]
        for p in parts:
            mx.fn_load(self.fd, p)
            mx.fn_load(self.fm, p)
        if warm:
            w_items = self.items(len(parts), len(parts))
            for kind, _, t in w_items:
                self.submit(mx.MX_PART_ANY, kind, t)
            for _, _, t in w_items:
                mx.fn_wait(t)
        items = self.items(n_tasks // 2, n_tasks - n_tasks // 2)
        W = resize_every if resize_every else len(items)
        waves = [items[i:i + W] for i in range(0, len(items), W)]
        res_by_wave, resize_ms, use_b = {}, [], False
        h0 = time.perf_counter()
        for w, wave in enumerate(waves):
            if w >= 2:
                res_by_wave[w - 2] = [mx.fn_wait(t) for _, _, t in waves[w - 2]]
                if resize_every and len(sizes) == len(LAYOUT_B):
                    use_b = not use_b
                    resize_ms += self.apply_layout(parts, LAYOUT_B if use_b else sizes)
            for kind, _, t in wave:
                self.submit(mx.MX_PART_ANY, kind, t)
        for w in range(len(waves)):
            if w not in res_by_wave:
                res_by_wave[w] = [mx.fn_wait(t) for _, _, t in waves[w]]
        wall = time.perf_counter() - h0
        res = [r for w in range(len(waves)) for r in res_by_wave[w]]
        info = [mx.part_query(p) for p in parts]
        for p in parts:
            self.destroy(p)
        return {"items": items, "results": res, "resize_ms": resize_ms, "wall_s": wall,
                "parts_info": info}


FILL7 = LAYOUTS_FILL[7]
