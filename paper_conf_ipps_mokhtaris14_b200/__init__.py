"""B200-native BigKernel streaming path (Mokhtari & Stumm, IPDPS 2014).

The product is libbk.so (include/bk.h): sm_100a kernels + C++ runtime. This package holds only
the thin ctypes binding (bk.py). It never imports the oracle and has no CPU fallback.
"""
from .bk import (BK_GATHER_AUTO, BK_GATHER_DENSE, BK_GATHER_ZC, BK_K_GREP, BK_K_GROUPBY, BK_K_KMEANS,
                 BK_K_LAYOUT_DUMP, BK_K_PARTITION, BK_K_WORDCOUNT, BkError, Context, bk_create, bk_destroy,
                 bk_get_stats, bk_register_segments, bk_run)

__all__ = ["Context", "BkError", "bk_create", "bk_register_segments", "bk_run", "bk_destroy", "bk_get_stats",
           "BK_K_WORDCOUNT", "BK_K_GREP", "BK_K_KMEANS", "BK_K_PARTITION", "BK_K_GROUPBY", "BK_K_LAYOUT_DUMP",
           "BK_GATHER_AUTO", "BK_GATHER_ZC", "BK_GATHER_DENSE"]
