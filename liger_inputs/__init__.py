"""Seeded synthetic input generators shared by the oracle, the tests and bench.py.

This package holds NO arithmetic of the method (no layer math, no scheduling):
only model shapes (Table 1; BASELINE.json configs), the
counter-based weight generator "C0" and the Poisson
request-trace generator.

The CUDA library implements the same counter-based generator independently in
`c0_fill_kernel` (`paper_conf_ppopp_duwjchcl24_b200/csrc/norm.cu`); tests check the two agree
bit-for-bit.  Nothing here imports `oracle/` or the CUDA binding.
"""
from .configs import CONFIGS, ModelConfig, get_config  # noqa: F401
from .c0 import (  # noqa: F401
    mix64, c0_uniform, c0_values, bf16_rne, weight_exp, emb_exp, layer_tensor,
    global_tensor, layer_activation, KIND, GLOBAL_ID,
)
from .traces import make_trace  # noqa: F401
