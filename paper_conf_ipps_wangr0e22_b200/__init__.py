"""B200-native MICCO correlator engine (dblp/paper_conf_ipps_wangr0e22).

The product is ``libmicco.so`` (C-ABI in include/micco.h; CUDA kernels for
sm_100a + a C++ builder/planner/scheduler/executor).  ``micco`` is the thin
ctypes binding.  Build with ``python tools/build.py``.
"""
from .micco import (Context, MiccoError, load_workload, micco_add_graph, micco_add_hadron_node,  # noqa: F401
                    micco_add_hadron_nodes_synth, micco_create, micco_debug_schedule, micco_destroy,
                    micco_execute, micco_get_correlator, micco_get_graph_value, micco_get_stats, micco_plan,
                    micco_release_cache, micco_nccl_unique_id, micco_set_nccl_id, micco_plan_ops, micco_dag,
                    micco_plan_stages, micco_predict_bounds, micco_probe_fp64_peak, micco_set_policy, BOUND_MODES,
                    lib, EXPORTS)
