"""deepplan-b200: B200-native DeepPlan cold-start inference hot path.

A thin ctypes binding over ``libdeepplan.so`` (C-ABI declared in ``include/deepplan.h``).
Argument marshalling only: every step of the path -- planning, the pinned weight arena,
transfers, event gating and every kernel -- runs in the native library.  PyTorch supplies
device memory and streams.  There is no CPU or Python fallback: if the extension is not
built, importing this package raises.
"""
from ._lib import (  # noqa: F401
    DHA, LOAD, MODES, UNIT_KINDS, Context, DeepPlanError, Model, attention, embed, host_alloc, host_free,
    layernorm, lib, linear, plan_exhaustive, plan_generate, plan_partition, plan_simulate, serve_run,
    peer_unique_id, measure_h2d, transfer_schedule, config_units, pt_forward, plan_resident_bytes,
    device_numa_node, host_numa_node, host_alloc_node, measure_h2d_concurrent, select_secondaries, attention_tc, gemm_tc,
)

__all__ = [
    "DHA", "LOAD", "MODES", "UNIT_KINDS", "Context", "DeepPlanError", "Model", "attention", "embed",
    "host_alloc", "host_free", "layernorm", "lib", "linear", "plan_exhaustive", "plan_generate",
    "plan_partition", "plan_simulate", "serve_run", "peer_unique_id", "measure_h2d", "transfer_schedule",
    "config_units", "pt_forward", "plan_resident_bytes", "device_numa_node", "host_numa_node", "host_alloc_node",
    "measure_h2d_concurrent", "select_secondaries", "attention_tc", "gemm_tc",
]
