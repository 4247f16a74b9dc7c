"""B200-native gSWORD hot path: WanderJoin / Alley random-walk subgraph-count
estimation with Horvitz-Thompson aggregation (§2.2, §3; Eq. 1).

The compute path is libgsword.so (sm_100a CUDA kernels + C++ host, C ABI in
include/gsword.h); this package is its thin binding plus the multi-GPU driver.
"""
from .gsword import (ALLEY, FILTER_LABEL, FILTER_LDF, FILTER_NLF, METHODS, OPT_AUTOTUNE, OPT_BLOCKS_PER_SM,
                     OPT_BLOOM, OPT_BLOOM_BITS, OPT_CHUNK, OPT_COOP_THRESHOLD, OPT_EDGE_SET, OPT_FAULT_QUEUE, OPT_FILTER,
                     OPT_L2_PERSIST, OPT_OCCUPANCY, OPT_REFILL_MIN, OPT_SCHEDULE, OPT_STREAMING, OPT_THREADS,
                     OPT_TRAWL_WARP, OPT_VARIANT, ORDER_QUICKSI, ORDER_TRIAL, RECORD_DTYPE, SCHED_INHERIT, SCHED_REFILL,
                     SCHED_SAMPLE_SYNC, TRAWL_DTYPE, VARIANT_ALLEY_DUPCHECK_POST, VARIANT_WJ_PARENT_FIRST, WJ,
                     Context, GswordError, check_graph, finalize, plan_query, qerror, quicksi_order, version)

__all__ = ["ALLEY", "FILTER_LABEL", "FILTER_LDF", "FILTER_NLF", "METHODS", "OPT_AUTOTUNE", "OPT_BLOCKS_PER_SM",
           "OPT_BLOOM", "OPT_BLOOM_BITS", "OPT_CHUNK", "OPT_COOP_THRESHOLD", "OPT_EDGE_SET", "OPT_FAULT_QUEUE", "OPT_FILTER",
           "OPT_L2_PERSIST", "OPT_OCCUPANCY", "OPT_REFILL_MIN", "OPT_SCHEDULE", "OPT_STREAMING", "OPT_THREADS",
           "OPT_TRAWL_WARP", "OPT_VARIANT", "ORDER_QUICKSI", "ORDER_TRIAL", "RECORD_DTYPE", "SCHED_INHERIT", "SCHED_REFILL",
           "SCHED_SAMPLE_SYNC", "TRAWL_DTYPE", "VARIANT_ALLEY_DUPCHECK_POST", "VARIANT_WJ_PARENT_FIRST", "WJ",
           "Context", "GswordError", "check_graph", "finalize", "plan_query", "qerror", "quicksi_order", "version"]
