"""Model shapes used by the benchmarks and tests.

OPT-30B / OPT-66B / GLM-130B come from PAPER.md Table 1 (layers,
heads, hidden).  FFN = 4*hidden ("GLM-130B has the same layer setup as GPT-3",
P:280; OPT uses 4h).  OPT-13B and the tiny config come from BASELINE.json
`configs`.  Vocabulary sizes are not in the paper (reading R14):
OPT 50272, GLM-shaped 150528.  Activation (reading R13): ReLU for OPT,
tanh-GELU for tiny and GLM-shaped.
"""
from dataclasses import dataclass, asdict


@dataclass(frozen=True)
class ModelConfig:
    name: str
    n_layers: int
    hidden: int
    n_heads: int
    ffn: int
    vocab: int
    max_pos: int
    act: str          # "relu" | "gelu_tanh"
    ln_eps: float = 1e-5

    @property
    def head_dim(self) -> int:
        return self.hidden // self.n_heads

    def asdict(self):
        return asdict(self)


CONFIGS = {
    # BASELINE.json configs[0]: 2 layers, hidden 256, 4 heads (d=64), TP=2,
    # batch 2, prompt 32 + 8 decode.  vocab 512 is a proposal.
    "tiny": ModelConfig("tiny", 2, 256, 4, 1024, 512, 64, "gelu_tanh"),
    # BASELINE.json configs[1]
    "opt-13b": ModelConfig("opt-13b", 40, 5120, 40, 20480, 50272, 2048, "relu"),
    # Table 1
    "opt-30b": ModelConfig("opt-30b", 48, 7168, 56, 28672, 50272, 2048, "relu"),
    # Table 1
    "opt-66b": ModelConfig("opt-66b", 64, 9216, 72, 36864, 50272, 2048, "relu"),
    # Table 1, GPT-3 layer setup
    "glm-130b": ModelConfig("glm-130b", 70, 12288, 96, 49152, 150528, 2304, "gelu_tanh"),
}


def get_config(name: str, n_layers: int | None = None) -> ModelConfig:
    c = CONFIGS[name]
    if n_layers is not None and n_layers != c.n_layers:
        d = c.asdict()
        d["n_layers"] = n_layers
        d["name"] = f"{c.name}[L={n_layers}]"
        c = ModelConfig(**d)
    return c
