"""Seeded synthetic inputs (SPN graphs + data) shared by the oracle tests and
the CUDA path.  Holds none of the method's arithmetic: structure, parameters
and sampling only (task rule ③)."""
from .graph import (FlatSPN, GraphBuilder, disjoint_union, GAUSSIAN,
                    CATEGORICAL, HISTOGRAM, SUM, PRODUCT, KIND_NAMES)
from .generators import (toy_spn, speaker_spn, speaker_set, tiny_discrete_spn,
                         tiny_gaussian_spn, rat_spn, rat_counts, CONFIGS,
                         config_graph)
from .sampling import (ancestral_sample, add_outliers, nan_mask, toy_data,
                       uniform_chunked)

__all__ = [n for n in dir() if not n.startswith("_")]
