"""paper_conf_sc_bradleyab25_b200 -- B200-native Fringe-SGC (SC'25).

The counting path is ``libfsgc.so`` (include/fsgc.h, CUDA for sm_100a); this
package is its thin Python binding.  Importing it loads the library and fails
loudly if it has not been built -- there is no CPU fallback.
"""
from ._lib import FsgcError, LIB_PATH, EXPORTS  # noqa: F401
from .api import (  # noqa: F401
    Graph, Pattern, CountResult, fsgc_load_graph, fsgc_compile_pattern, compile_named,
    fsgc_count, fsgc_count_distributed, combine_partials, fsgc_num_roots, fsgc_finalize,
    Plan, fsgc_plan_create,
)

__all__ = [
    "Graph", "Pattern", "CountResult", "FsgcError", "fsgc_load_graph", "fsgc_compile_pattern",
    "compile_named", "fsgc_count", "fsgc_count_distributed", "fsgc_num_roots", "fsgc_finalize",
]
