"""CPU ORACLE — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct NumPy (float64) implementation of what the
multiplexed small-function hot path computes:

  * decode.py   — Llama-style greedy decode task (C2/C3)            [pinned]
  * mpnn.py     — IP-emulator message-passing inference (C4)        [pinned by
                  closed forms / invariants / dense reformulation; the
                  architecture itself is our reading A22 of PAPER.md §3.1
                  step (4): *parity vs the paper is unpinned*]
  * sched.py    — deterministic placement simulator + canonical trace (C5)
  * invariants.py — I1-I6 (C6)
  * cost.py     — algorithmic bytes / flops per task (D0) and default
                  placement cost (C5)
  * numerics.py — bf16 round-to-nearest-even (the KV rounding point, A16)

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s cpu_baseline /
`--impl reference` legs may import this package. The product path
(`paper_conf_sc_dhakalrwercfm23_b200`, `include/`, `csrc/`) never imports,
links or executes it, and it shares no code with the CUDA path: the only
shared module is `workloads/` (seeded integer generators, no arithmetic of
the method).

Citations: `P:NNN` = line of PAPER.md (Dhakal et al., SC-W 2023), with the
section it falls in; `C1..C7`, `A1..A27` = SURVEY.md §8(c) items.
"""
