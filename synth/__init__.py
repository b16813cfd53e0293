"""Seeded synthetic fp32 fields shaped like the paper's datasets (Table 2,
P:864-872).  Harness code shared by tests and bench: it contains none of
the method's arithmetic (no quantisation, prediction, encoding or scan),
so it is the one module both the oracle side and the CUDA side may use.

Recipes: calibrated against what the paper states about
each dataset -- smoothness (Fig 6), value ranges (artifact,
P:1923), sparsity growing over time for RTM, zero blocks
(P:370-375).  Torch is used only as an array library; every generator
takes a ``device`` so large fields are built directly in HBM.
"""
from .fields import (  # noqa: F401
    CONFIGS,
    DATASET_RELS,
    DATASETS,
    dataset_field,
    field_for_config,
    hacc_like,
    hurricane_like,
    nyx_like,
    qmcpack_like,
    cesm_like,
    rtm_like,
    smooth1d,
)
