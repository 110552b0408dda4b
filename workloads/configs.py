"""Model shapes, seeds and workload recipes.

Pure data: no arithmetic of the method lives here. Both the oracle and the
harness read these shapes; the CUDA library receives them through the C ABI
(mx_decode_cfg / mx_mpnn_cfg).
"""
from __future__ import annotations

from dataclasses import dataclass, asdict, replace


@dataclass(frozen=True)
class DecodeCfg:
    """Llama-style decoder shape (ambiguity register A8, A12, A13)."""
    name: str
    n_layers: int
    d_model: int
    n_heads: int
    n_kv_heads: int
    head_dim: int
    d_ff: int
    vocab: int
    max_seq: int = 64
    rms_eps: float = 1e-5
    rope_theta: float = 10000.0
    seed: int = 0

    @property
    def q_dim(self) -> int:
        return self.n_heads * self.head_dim

    @property
    def kv_dim(self) -> int:
        return self.n_kv_heads * self.head_dim

    def with_layers(self, n: int) -> "DecodeCfg":
        return replace(self, n_layers=n, name=f"{self.name}-L{n}")

    def asdict(self):
        return asdict(self)


@dataclass(frozen=True)
class MpnnCfg:
    """IP-emulator message-passing network shape."""
    name: str = "mpnn"
    n_atom_types: int = 8
    n_bond_types: int = 4
    hidden: int = 128
    steps: int = 3
    seed: int = 0x3D01

    def asdict(self):
        return asdict(self)


# configs[0]: tiny decoder (2 layers, d=256, vocab 1k)  -- A13: H4 hd64 d_ff 768
TINY = DecodeCfg("tiny", n_layers=2, d_model=256, n_heads=4, n_kv_heads=4, head_dim=64,
                 d_ff=768, vocab=1024, seed=0x7111)
# configs[1]: GPT-2-small-shaped Llama block -- A12
GPT2S = DecodeCfg("gpt2s", n_layers=12, d_model=768, n_heads=12, n_kv_heads=12, head_dim=64,
                  d_ff=2048, vocab=50257, seed=0x6732)
# configs[2]: 7B-Llama-shaped -- A8 (public Llama-2-7B dims)
LLAMA7B = DecodeCfg("llama7b", n_layers=32, d_model=4096, n_heads=32, n_kv_heads=32,
                    head_dim=128, d_ff=11008, vocab=32000, seed=0x7B00)
# a ragged shape used only by parity tests: nothing a multiple of 256, odd vocab, GQA
RAGGED = DecodeCfg("ragged", n_layers=2, d_model=264, n_heads=6, n_kv_heads=2, head_dim=32,
                   d_ff=712, vocab=1031, seed=0x5EED)

# split-K shape used only by parity tests: at batch 8 the inputs of width d_model
# (2056 -> 2 segments, ragged second) and d_ff (2600 -> 2 segments) exceed the
# 64 KiB activation staging, q_dim 512 does not; GQA 8/2, separate attention phase
SPLITK = DecodeCfg("splitk", n_layers=2, d_model=2056, n_heads=8, n_kv_heads=2, head_dim=64,
                   d_ff=2600, vocab=1031, seed=0x5A17)

MPNN = MpnnCfg()

DECODE_CFGS = {c.name: c for c in (TINY, GPT2S, LLAMA7B, RAGGED, SPLITK)}

# Default seeds
SEED_PROMPT = 0xC0FFEE
SEED_GRAPH = 0x6A5
SEED_SHUFFLE = 42

# Decode tensor ids (C1)
T_EMBED = 0
T_WQ, T_WK, T_WV, T_WO, T_WGATE, T_WUP, T_WDOWN, T_GATTN, T_GMLP = range(9)


def layer_tid(layer: int, which: int) -> int:
    return 16 * (layer + 1) + which


def gfinal_tid(cfg: DecodeCfg) -> int:
    return 16 * (cfg.n_layers + 1)


def lmhead_tid(cfg: DecodeCfg) -> int:
    return 16 * (cfg.n_layers + 1) + 1


# MPNN tensor ids (C1): 0 E_atom, 1-4 W_b, 5 U, 6 c, 7 W1, 8 c1, 9 w2, 10 c2
M_EATOM, M_WB0, M_U, M_C, M_W1, M_C1, M_W2, M_C2 = 0, 1, 5, 6, 7, 8, 9, 10


# Workload recipes
@dataclass(frozen=True)
class DecodeWorkload:
    cfg: DecodeCfg
    n_tasks: int
    batch: int
    prompt_len: int
    gen_len: int


C1 = DecodeWorkload(TINY, n_tasks=4, batch=1, prompt_len=8, gen_len=16)
C2 = DecodeWorkload(GPT2S, n_tasks=700, batch=1, prompt_len=16, gen_len=32)
C3 = DecodeWorkload(LLAMA7B, n_tasks=100, batch=1, prompt_len=16, gen_len=32)
MPNN_MOLS_PER_TASK = 1024

# D0 partition layouts on 148 SMs. The library splits a B200 into 37 groups of
# 4 SMs (green-context split ignoring SM co-scheduling; reading R8),
# so "fill" layouts (MPS-like, primary) use all 148 SMs and "equal" layouts
# (MIG-like fixed slices, §5.2) use identical sizes.
LAYOUTS_FILL = {
    1: [148],
    2: [76, 72],
    4: [40, 36, 36, 36],
    7: [24, 24, 20, 20, 20, 20, 20],
    14: [12] * 9 + [8] * 5,
    # finer than the paper's 1-4 processes / BASELINE's 14 (extra sweep points)
    18: [8] * 18 + [4],
    37: [4] * 37,
}
LAYOUTS_EQUAL = {
    1: [148],
    2: [72, 72],
    4: [36] * 4,
    7: [20] * 7,
    14: [8] * 14,
}
