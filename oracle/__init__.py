"""CPU oracle for the maximum-clique hot path -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
`--impl reference` leg may import this package.  The product path
(paper_conf_ipps_geilpo23_b200) never imports it and fails loudly when its
CUDA library is missing.  See mce_oracle.c for the passage each function
follows and tests/test_oracle.py for the pins.
"""

from .oracle import (  # noqa: F401
    build,
    count_max_cliques,
    core_numbers,
    default_threshold,
    greedy,
    is_clique,
    kclique_counts,
    max_cliques,
)
