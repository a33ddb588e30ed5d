"""B200-native exhaustive co-scheduling configuration search (sm_100a).

Hot path of Weaver et al., "Granularity- and Interference-Aware GPU Sharing
with MPS" (SC'24 workshops): score every configuration of N profiled
workflows on G GPUs (MPS client groups x active-thread levels) for
throughput and energy efficiency, return the best per product metric and
the exact Pareto set.  C ABI: include/sched.h; kernels: csrc/.
"""
from .sched import (Scheduler, SearchResult, SchedError, Pick, count, unrank, rank, merge,  # noqa: F401
                    version, lib, PER_CLIENT, PER_GPU, EXPORTS)
from .resume import search_resumable, CoverageError  # noqa: F401,E402
