"""B200-native gSWORD hot path: WanderJoin / Alley random-walk subgraph-count
estimation with Horvitz-Thompson aggregation (§2.2, §3; Eq. 1).

The compute path is libgsword.so (sm_100a CUDA kernels + C++ host, C ABI in
include/gsword.h); this package is its thin binding plus the multi-GPU driver.
"""
from .gsword import (TRAWL_DTYPE, ORDER_QUICKSI, ORDER_TRIAL, quicksi_order, ALLEY, METHODS, OPT_BLOCKS_PER_SM, OPT_BLOOM, OPT_CHUNK, OPT_COOP_THRESHOLD, OPT_EDGE_SET, OPT_FILTER, OPT_SCHEDULE, OPT_REFILL_MIN, OPT_AUTOTUNE, OPT_BLOOM_BITS, OPT_STREAMING, OPT_VARIANT, OPT_OCCUPANCY, VARIANT_WJ_PARENT_FIRST, VARIANT_ALLEY_DUPCHECK_POST, SCHED_REFILL, SCHED_SAMPLE_SYNC, SCHED_INHERIT, FILTER_LABEL, FILTER_LDF, FILTER_NLF, OPT_L2_PERSIST,
                     OPT_THREADS, RECORD_DTYPE, WJ, Context, GswordError, check_graph, finalize, plan_query,
                     qerror, variance_tolerance, version)

__all__ = ["TRAWL_DTYPE", "ORDER_QUICKSI", "ORDER_TRIAL", "quicksi_order", "ALLEY", "WJ", "METHODS", "Context", "GswordError", "RECORD_DTYPE", "check_graph", "finalize",
           "plan_query", "qerror", "variance_tolerance", "version", "OPT_BLOCKS_PER_SM", "OPT_BLOOM", "OPT_CHUNK", "OPT_EDGE_SET", "OPT_FILTER", "OPT_SCHEDULE", "OPT_REFILL_MIN", "OPT_AUTOTUNE", "OPT_BLOOM_BITS", "OPT_STREAMING", "OPT_VARIANT", "OPT_OCCUPANCY", "VARIANT_WJ_PARENT_FIRST", "VARIANT_ALLEY_DUPCHECK_POST", "SCHED_REFILL", "SCHED_SAMPLE_SYNC", "SCHED_INHERIT", "FILTER_LABEL", "FILTER_LDF", "FILTER_NLF",
           "OPT_COOP_THRESHOLD", "OPT_L2_PERSIST", "OPT_THREADS"]
