"""Seeded synthetic inputs shared by the oracle and the GPU path (input construction only)."""
from .corpus import (  # noqa: F401
    Corpus, dictionary, patterns, gen_bytes, make_corpus, write_file, NDICT, NPAT,
    SEED_FILE16M, SEED_CORPUS, SEED_DICT, SEED_PLANTS, SEED_AMR, SEED_SIGNAL, amr_levels, signal_blocks, perm_inputs,
)
