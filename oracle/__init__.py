"""ORACLE -- test infrastructure only.

A plain, slow, obviously-correct CPU model of MPress's D2D stripe swap
(Zhou et al., HPCA'23), written from the paper (/root/reference/PAPER.md, cited
``P:<line>``) and the readings R1..R21 listed in DESIGN.md §3.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_hpca_zhouwylbyx23_b200``, ``include/mpress.h``, the CUDA
kernels) never imports, links or executes it, and shares no code with it: the
two meet only through the seeded generators in ``synth/``.

Modules
  plan       -- the stripe planner (greedy unit apportionment, §III-C)
  bytemodel  -- byte-exact model of swap-out / swap-in
  brute      -- exhaustive minimum-makespan search for tiny inputs
  partition  -- sequential multi-source stash reservation (reading R12)
  global_plan -- NEXT-1: joint multi-exporter assignment (Fig. 6, R23)

Pins (tests/test_oracle.py): the paper's worked 1:2 ratio (golden G2),
equal striping on symmetric links, brute-force optimality of the score
(P:213), capacity / coverage invariants (Fig. 6 line 3), the
bandwidth-proportionality bound, round-trip identity, and a
hand-checked golden plan (G1).  No function here is "parity unpinned".
"""
from .plan import (  # noqa: F401
    ALIGN, DEFAULT_GRANULE, PlanError, ERR_ARG, ERR_NO_SPACE, plan, plan_from_units, virtual_layout,
)
from .bytemodel import swap_out, swap_in, stash_sizes  # noqa: F401
from .brute import brute_force_makespan, makespan  # noqa: F401
from .partition import sequential_partition  # noqa: F401
from .global_plan import brute_force_global, scan_global, assignment_time  # noqa: F401
from .mapping import mapping_search  # noqa: F401
