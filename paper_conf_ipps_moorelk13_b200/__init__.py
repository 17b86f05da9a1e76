"""B200-native (sm_100a) spatial-domain NCC: template matching and PIV.

The product is libncc_b200.so (C ABI in include/ncc.h); this package only binds it.
Import is light: the CUDA library is loaded on first use and its absence is an error,
never a fallback.
"""
from ._native import (NccError, NccProblem, make_problem, ncc_match, ncc_match_host, ncc_match_rois,  # noqa: F401
                      ncc_plan_create,
                      ncc_plan_destroy, ncc_plan_query, ncc_plan_timing, ncc_specialize, ncc_status_string, piv_correlate,
                      piv_correlate_ex, piv_correlate_host)

__all__ = ["NccError", "NccProblem", "make_problem", "ncc_plan_create", "ncc_match", "ncc_match_rois",
           "piv_correlate",
           "piv_correlate_ex", "ncc_match_host", "piv_correlate_host", "ncc_plan_destroy", "ncc_plan_query",
           "ncc_plan_timing", "ncc_specialize", "ncc_status_string"]
