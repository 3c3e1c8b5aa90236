"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This package holds NONE of the method's arithmetic (no digitisation, no MLP, no argmax):
it draws traces, raw feature records and random-init weights. Everything is seeded
(numpy PCG64), so the oracle and the CUDA path see byte-identical inputs.

* Traces follow §7.1: "an exponential distribution for inter-arrival time,
  a lognormal distribution for I/O size and a uniform distribution for I/O offset", with
  the Table 4 device profiles and "rerating".
* Raw records are what the feature registry captures on issue / completion
  (Fig. 4/5), computed by exact event simulation (tracesim.c).
* Weights are random init (no trained LinnOS weights are published).
The full recipe and every silent-parameter reading is in DESIGN.md §5.
"""
from .gen import (  # noqa: F401
    PROFILES,
    PROFILE_ORDER,
    ARCH_WIDTHS,
    blob_floats,
    device_trace,
    multi_device_trace,
    weights,
    raw_weights,
    edge_raw,
    workload,
    CONFIGS,
)
