"""Seeded synthetic inputs shared by the oracle tests, the CUDA parity tests and bench.py.

This package holds NONE of the method's arithmetic (no sampling, no dedup, no
time encoding, no attention): it only draws edge streams, feature tables and
model parameters from seeded numpy generators, in the shapes of the paper's
workloads (Table 2) and BASELINE.json's configs.
Both `oracle/` and the product path consume its outputs; it imports neither.
"""
from .configs import CONFIGS, StreamConfig, ModelConfig, get_config  # noqa: F401
from .streams import make_stream, negatives, Stream  # noqa: F401
from .params import make_params, param_count  # noqa: F401
