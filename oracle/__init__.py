"""TeMCO oracle -- TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU implementation of what the TeMCO hot path
computes (PAPER.md = /root/reference/PAPER.md, cited as P:L<line>):

  * graph.py   -- decomposition expansion (O1: Eq. (2)) and
                  shape / size / FLOP inference,
  * rewrite.py -- tensor liveness and skip detection (Alg. 1),
                  FindReduced / Compare / Peak / IsLConv (Alg. 2),
                  Overhead, COPY + InsertBefore
                  (P:L213-214), DCE, activation-layer fusion grouping
                   with the layer transformations,
                  the merged-fconv CSE (reading R37) and the memory-optimal
                  re-scheduling of S (reading R38),
                  and the peak internal-tensor accounting (Eq. (3)/(4),
                  P:L109-120),
  * ops.py     -- fp64 direct-loop convolution / BN / ReLU / pools / linear,
  * execute.py -- the unfused decomposed model and the TeMCO-transformed model.

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s `cpu_baseline` /
`--impl reference` legs may import anything under `oracle/`.  The oracle
shares no code with the CUDA path (`paper_conf_icpp_songljkj0024_b200/`);
it reads only the seeded inputs of `workloads/`.

Parity status per function is listed in DESIGN.md ("Oracle pins"); the paper's
percentages (75.7 % etc.) are "parity unpinned" (unknown model variants,
trained weights and allocator accounting).
"""
from .graph import expand, Node, DTYPE_BYTES  # noqa: F401
from .rewrite import plan, Plan, liveness, find_reduced, peak_fn, peak_bytes  # noqa: F401
from .execute import run_unfused, run_temco, run_decomposed_order  # noqa: F401
