"""B200-native graphB+ balancing hot path (Alabandi et al., SC'21).

The product is libgraphb.so (include/graphb.h, csrc/*.cu, sm_100a); this
package is its thin Python binding.  See DESIGN.md.
"""
from . import graphb  # noqa: F401
from .graphb import (GraphBError, balance, balance_given_tree, balance_host,  # noqa: F401
                     balance_range, free, graph_info, load_csr, load_graph, set_option,
                     stats, tree_debug, tree_stats)

__all__ = ["graphb", "GraphBError", "load_csr", "load_graph", "balance", "balance_host",
           "balance_range", "free", "tree_debug", "balance_given_tree", "set_option",
           "stats", "tree_stats", "graph_info"]
