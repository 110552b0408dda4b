"""Writes the frozen generator fixtures under tests/golden/.

Calls only `workloads/` (the seeded integer generators of SURVEY.md §8(c) C1)
and `oracle/`; never the CUDA path. Re-run only when the recipe changes, and
cite the reason in the commit message.
"""
import os
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.dirname(os.path.dirname(HERE)))

from workloads.inputs import molecule_slow  # noqa: E402


def main():
    types, edges = molecule_slow(1, 0)
    with open(os.path.join(HERE, "molecule_task1_mol0.txt"), "w") as f:
        f.write("# First molecule of task 1 (graph seed 0x6A5), SURVEY.md §8(c) C1 recipe.\n")
        f.write("# line 1: atom types; line 2: edges u,v,bond in generation order.\n")
        f.write(" ".join(map(str, types)) + "\n")
        f.write(" ".join(f"{u},{v},{b}" for u, v, b in edges) + "\n")


if __name__ == "__main__":
    main()
