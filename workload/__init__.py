"""Seeded synthetic inputs (the only module shared by oracle tests and the GPU harness).

Holds no SNICIT arithmetic; see sdgc.py for the recipe and its citations.
"""
from .sdgc import (BASE_SEED, CONFIGS, CirculantNetwork, gen_circulant, SNICIT_SDGC, SNICIT_MEDIUM, Network, connections,  # noqa: F401
                   gen_inputs, gen_medium_inputs, gen_medium_network, gen_network, medium_t,
                   radix_strides)
