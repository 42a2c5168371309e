"""Multigrain oracle — TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU (numpy, fp64) statement of what the
compound sparse attention forward computes, written from the paper
(/root/reference/PAPER.md, cited as ``P:<line>``) and the readings recorded in
DESIGN.md §3 / SURVEY.md §8(c).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
leg / ``--impl reference`` arm may import anything from this package. The
product path (``paper_conf_iiswc_lica22_b200``) never imports it, and this
package never imports the product path: the two share no code. The only common
module is ``workloads`` (seeded input generators, no method arithmetic).

Modules
* ``oracle.mask``       — the union mask M (O-2): local ∨ global-row ∨ global-col ∨ extra.
* ``oracle.plan``       — the canonical coarse/fine/dense-row partition (O-3).
* ``oracle.attention``  — dense masked attention (O-4), CSR reference (O-5),
                          partitioned LSE-merged reference (O-6), staged S/P (O-7),
                          and per-row evaluation for sampled parity at full size.

Parity pins (tests/test_oracle_*.py): closed-form counts, the P:185 block
ratios, a hand-worked example (tests/golden/worked_example_L8.json),
brute force on tiny L, library special cases (torch SDPA in fp64), and
invariants. No oracle function is "parity unpinned".
"""
from .mask import ExtraIndex, union_mask_dense, mask_rows, mask_row_cols, global_flags
from .plan import CanonicalPlan, canonical_plan
from .attention import (
    dense_masked_attention, csr_reference, partitioned_reference, staged_intermediates,
    attention_rows, head_inputs_f64, useful_flops,
)

__all__ = [
    "ExtraIndex", "union_mask_dense", "mask_rows", "mask_row_cols", "global_flags",
    "CanonicalPlan", "canonical_plan",
    "dense_masked_attention", "csr_reference", "partitioned_reference", "staged_intermediates",
    "attention_rows", "head_inputs_f64", "useful_flops",
]
