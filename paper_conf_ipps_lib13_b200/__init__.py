"""agraph — adaptive BFS/SSSP frontier engine for B200 (Li & Becchi, IPDPS 2013, re-designed for sm_100a).

The product is ``libagraph.so`` (C ABI, ``include/agraph.h``); ``agraph`` is its ctypes binding.
"""
from . import agraph  # noqa: F401
from .agraph import Graph, Policy, policy_default, select, AgError  # noqa: F401
