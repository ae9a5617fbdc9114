"""Seeded synthetic workloads shared by the oracle tests, the GPU tests and bench.py.

This package holds NO arithmetic of the Skipper method (no LIF update, no
surrogate, no percentile, no GEMM).  It only describes network topologies
 and draws seeded random inputs:

* grid-quantised weights  w = j * 2**-e, |j| <= 255   (SURVEY.md §8(c) "exactness protocol")
* Poisson rate-coded input spikes  o0_t = [u_t < x * r_t]   (reading 18)
* DVS-shaped event frames (synthetic stand-in, reading 18)
* uniform class labels

Both sides (oracle/ and the CUDA path) receive the exact same arrays.
"""
from .configs import NETS, net_config, workload, WORKLOADS  # noqa: F401
from .inputs import (  # noqa: F401
    grid_weights, poisson_frames, dvs_frames, labels, make_inputs, make_weights, envelope, weight_shape,
)
