"""B200-native Smith-Waterman/Gotoh protein database search with the PSS/WA scheduler of
Mendonca & Melo (IPDPSW 2013).  The compute path is libsw (csrc/, C-ABI in include/sw.h);
this package is its thin Python binding plus the multi-process (torchrun) glue.
"""
from .binding import (Database, Scheduler, SearchResult, SwError, lib, EXPORTS, Master, Slave, chrome_trace,  # noqa: F401
                      grant_timeline,
                      SW_TASK_READY, SW_TASK_EXECUTING, SW_TASK_FINISHED)
from . import _build  # noqa: F401

__all__ = ["Database", "Scheduler", "SearchResult", "SwError", "lib", "EXPORTS", "chrome_trace", "grant_timeline"]
