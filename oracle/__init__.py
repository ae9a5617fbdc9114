"""CPU oracle for Skipper SNN training (TEST INFRASTRUCTURE ONLY).

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s `cpu_baseline` /
`--impl reference` legs may import this package.  The product path
(`paper_conf_micro_singhslsknnd22_b200/`, `include/`) never imports, links or
executes anything under `oracle/`, and this package never imports the product.

What it computes (PAPER.md = /root/reference/PAPER.md, cited as P:<line>):

* Eq.1: LIF dynamics U_t = lam*U_{t-1} + W o^{l-1}_t - theta*o^l_{t-1},
  o_t = [U_t > theta], evaluated in float32 without FMA, in the order
  ((lam*U) + I) - theta*o  (the arithmetic contract of SURVEY.md §8(c)).
* Eq.2: surrogate-gradient BPTT with the reset detached, in float64,
  with bf16 rounding emulated at the GPU's GEMM-input points (delta before the
  dgrad/wgrad contractions, W everywhere).
* Sec. V (Fig. 5): temporal activation checkpointing with C segments,
  each recomputed exactly once per iteration.
* Sec. VI-A (Fig. 6): Skipper - SAM spike sums (Eq.4), per-segment
  p-th percentile SST_c (Eq.5), keep-if s_t > SST_c, compacted recompute chain
  (reading A of SURVEY.md §8(c) #14).
* Eq.3 / Eq.6 memory laws through an explicit ledger of the bytes it stores.
* Adam with torch.optim.Adam semantics.

Every function cites the passage it follows.  Pins (tests/test_oracle_*.py) tie
it to things other than itself: closed-form LIF spike trains, torch.autograd on
an explicitly unrolled network, scipy correlation, adjoint identities, the
paper's T=20/C=2 worked schedule, finite differences, torch.optim.Adam.
"""
from .numerics import bf16_round  # noqa: F401
from .layers import conv3x3, conv3x3_input_grad, conv3x3_weight_grad, pool2, pool2_T  # noqa: F401
from .lif import lif_step, surrogate_grad  # noqa: F401
from .skipper import spike_sum_threshold, keep_mask, kept_lists, ledger_model  # noqa: F401
from .bptt import StepConfig, StepResult, train_step, forward_first_pass  # noqa: F401
from .adam import adam_update  # noqa: F401
