"""B200-native two-pass min-wise Shingling (Wu & Kalyanaraman, gpClust, IPDPSW 2013).

The hot path lives in ``libshingle.so`` (hand-written sm_100a CUDA behind the
C ABI of ``include/shingle.h``); :mod:`.binding` is a thin ctypes layer with
the same function names.  Importing the package does not load the library;
the first binding call does, and raises if it is missing (no CPU fallback).
"""
from .binding import (ShingleGraph, SGError, group_by_shingle, report_dense_subgraphs,  # noqa: F401
                      shingle_graph_create, shingle_graph_destroy, shingle_graph_reset,
                      shingle_pass)

__all__ = ["ShingleGraph", "SGError", "shingle_graph_create", "shingle_pass", "group_by_shingle",
           "report_dense_subgraphs", "shingle_graph_reset", "shingle_graph_destroy"]
