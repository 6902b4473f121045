"""Seeded synthetic inputs (graph sets) for tests, smoke and bench.

Shared by the oracle side and the CUDA side; holds none of the method's
arithmetic (see graphset.py)."""
from .graphset import (ALLOC_DTYPE, ALL10, BATCH_SIZES, CONFIGS, MODELS, TABLE1_NODES, T_NEVER,  # noqa: F401
                       TAG_CONST, TAG_DANGLING, TAG_FP, TAG_GAP, TAG_NAMES, TAG_OPE, TAG_PTR, GraphSet,
                       make_graph_set)
