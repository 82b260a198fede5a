"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

This module holds NONE of the method's arithmetic (no clique search, no
k-core, no heuristic). It only produces undirected simple graphs in CSR form
from a counter-based random generator, so the same seed gives bit-identical
graphs on CPU (numpy / torch-CPU) and on the GPU (torch-CUDA).
"""

from .graphs import (  # noqa: F401
    CONFIGS,
    Graph,
    barabasi_albert,
    complete_graph,
    cycle_graph,
    erdos_renyi,
    from_edges,
    make_config,
    paley_graph,
    plant_cliques,
    rmat,
    turan_graph,
)
