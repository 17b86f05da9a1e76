"""ctypes binding of libncc_b200.so -- argument marshalling only.

Same names as the C ABI (include/ncc.h): ncc_plan_create, ncc_match, piv_correlate,
piv_correlate_ex, ncc_match_host, piv_correlate_host, ncc_plan_destroy, ncc_plan_query,
ncc_plan_timing, ncc_status_string.  Every computation happens inside the CUDA library;
if the library is missing this module raises -- there is no CPU fallback.
Tensors are torch tensors (device memory / pinned host memory); streams default to
torch's current stream on the plan's device.
"""
from __future__ import annotations

import ctypes
import os

PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(PKG, "libncc_b200.so")

NCC_OK = 0
STATUS = {0: "NCC_OK", 1: "NCC_ERR_INVALID_ARGUMENT", 2: "NCC_ERR_UNSUPPORTED", 3: "NCC_ERR_OUT_OF_MEMORY",
          4: "NCC_ERR_CUDA", 5: "NCC_ERR_COMPILE", 6: "NCC_ERR_WRONG_MODE"}
NCC_MODE_MATCH, NCC_MODE_PIV = 0, 1
NCC_SCORE_NCC, NCC_SCORE_SSD, NCC_SCORE_SAD = 0, 1, 2
NCC_SUBPIX_GAUSS3, NCC_SUBPIX_PARABOLA3, NCC_SUBPIX_NONE = 0, 1, 2
NCC_F_WRITE_SURFACE, NCC_F_GENERIC_KERNEL, NCC_F_NO_JIT, NCC_F_TIMING, NCC_F_CUDA_CORES = 1, 2, 4, 8, 16
FLAG_FLAT_TEMPLATE, FLAG_EDGE_Y, FLAG_EDGE_X, FLAG_PARABOLA_Y, FLAG_PARABOLA_X, FLAG_INVALID = 1, 2, 4, 8, 16, 32

EXPORTS = ["ncc_plan_create", "ncc_match", "ncc_match_rois", "piv_correlate", "piv_correlate_ex", "ncc_match_host",
           "piv_correlate_host", "ncc_plan_destroy", "ncc_status_string", "ncc_last_cuda_error",
           "ncc_plan_query", "ncc_plan_timing", "ncc_build_arch", "ncc_specialize"]


class NccProblem(ctypes.Structure):
    _fields_ = [("mode", ctypes.c_int32), ("score", ctypes.c_int32), ("subpix", ctypes.c_int32),
                ("image_h", ctypes.c_int32), ("image_w", ctypes.c_int32), ("image_pitch", ctypes.c_int64),
                ("tmpl_h", ctypes.c_int32), ("tmpl_w", ctypes.c_int32),
                ("search_y", ctypes.c_int32), ("search_x", ctypes.c_int32),
                ("step_y", ctypes.c_int32), ("step_x", ctypes.c_int32),
                ("batch", ctypes.c_int32), ("shard_rank", ctypes.c_int32), ("shard_count", ctypes.c_int32),
                ("flags", ctypes.c_uint32), ("n_templates", ctypes.c_int32), ("roi_h", ctypes.c_int32),
                ("roi_w", ctypes.c_int32)]


class NccPeak(ctypes.Structure):
    _fields_ = [("score", ctypes.c_float), ("u", ctypes.c_int32), ("v", ctypes.c_int32), ("flags", ctypes.c_uint32)]


class PivVector(ctypes.Structure):
    _fields_ = [("iy", ctypes.c_int32), ("ix", ctypes.c_int32), ("dy", ctypes.c_float), ("dx", ctypes.c_float),
                ("score", ctypes.c_float), ("flags", ctypes.c_uint32)]


class NccPlanInfo(ctypes.Structure):
    _fields_ = [("mode", ctypes.c_int32), ("U", ctypes.c_int32), ("V", ctypes.c_int32),
                ("u_begin", ctypes.c_int32), ("u_end", ctypes.c_int32), ("Ky", ctypes.c_int32),
                ("Kx", ctypes.c_int32), ("batch", ctypes.c_int32), ("outputs_per_call", ctypes.c_int64),
                ("flops_per_call", ctypes.c_double), ("specialized", ctypes.c_int32),
                ("variant_id", ctypes.c_int32), ("regs_per_thread", ctypes.c_int32),
                ("threads_per_block", ctypes.c_int32), ("smem_per_block", ctypes.c_int32),
                ("grid_x", ctypes.c_int32), ("grid_y", ctypes.c_int32), ("grid_z", ctypes.c_int32),
                ("launches_per_call", ctypes.c_int32), ("split", ctypes.c_int32),
                ("const_template", ctypes.c_int32), ("slabs", ctypes.c_int32),
                ("variant_name", ctypes.c_char * 96)]

    def as_dict(self):
        d = {k: getattr(self, k) for k, _ in self._fields_}
        d["variant_name"] = self.variant_name.decode()
        return d


class NccTiming(ctypes.Structure):
    _fields_ = [("prep_ms", ctypes.c_float), ("stats_ms", ctypes.c_float), ("numerator_ms", ctypes.c_float),
                ("finalize_ms", ctypes.c_float), ("total_ms", ctypes.c_float),
                ("numerator_launches", ctypes.c_int32)]


assert ctypes.sizeof(NccPeak) == 16 and ctypes.sizeof(PivVector) == 24

_lib = None


class NccError(RuntimeError):
    def __init__(self, status, where=""):
        msg = STATUS.get(status, str(status))
        if status == 4 and _lib is not None:
            msg += ": " + _lib.ncc_last_cuda_error().decode()
        super().__init__(f"{where}: {msg}" if where else msg)
        self.status = status


def lib():
    """Load the CUDA library; raise loudly if it is not built (no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"libncc_b200.so not found at {LIB_PATH}: run __graft_entry__.build() "
                               "(python -m paper_conf_ipps_moorelk13_b200.build). There is no CPU fallback.")
        L = ctypes.CDLL(LIB_PATH)
        P, V = ctypes.c_void_p, ctypes.c_void_p
        L.ncc_plan_create.argtypes = [ctypes.POINTER(NccProblem), ctypes.c_int, ctypes.POINTER(P)]
        L.ncc_match.argtypes = [P, P, P, ctypes.c_int64, P, P, V]
        L.ncc_match_rois.argtypes = [P, P, P, ctypes.c_int64, P, P, P, V]
        L.piv_correlate.argtypes = [P, P, P, P, V]
        L.piv_correlate_ex.argtypes = [P, P, P, P, P, V]
        L.ncc_match_host.argtypes = [P, P, P, ctypes.c_int64, P, P, V]
        L.piv_correlate_host.argtypes = [P, P, P, P, V]
        L.ncc_plan_destroy.argtypes = [P]
        L.ncc_status_string.argtypes = [ctypes.c_int]
        L.ncc_status_string.restype = ctypes.c_char_p
        L.ncc_last_cuda_error.restype = ctypes.c_char_p
        L.ncc_plan_query.argtypes = [P, P, ctypes.c_size_t]
        L.ncc_plan_timing.argtypes = [P, ctypes.POINTER(NccTiming)]
        L.ncc_build_arch.restype = ctypes.c_int32
        L.ncc_specialize.argtypes = [ctypes.POINTER(NccProblem), ctypes.c_char_p, ctypes.c_size_t,
                                     ctypes.POINTER(ctypes.c_int32)]
        for fn in EXPORTS:
            if fn not in ("ncc_status_string", "ncc_last_cuda_error", "ncc_build_arch"):
                getattr(L, fn).restype = ctypes.c_int
        _lib = L
    return _lib


def _check(st, where):
    if st != NCC_OK:
        raise NccError(st, where)


def _ptr(t):
    if t is None:
        return None
    if isinstance(t, int):
        return t
    return t.data_ptr()


def _stream(stream, device):
    if stream is None:
        import torch
        return torch.cuda.current_stream(device).cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def make_problem(mode=NCC_MODE_MATCH, image_h=0, image_w=0, image_pitch=None, tmpl_h=0, tmpl_w=0, search_y=0,
                 search_x=0, step_y=0, step_x=0, batch=1, shard_rank=0, shard_count=1, flags=0,
                 score=NCC_SCORE_NCC, subpix=NCC_SUBPIX_GAUSS3, n_templates=0, roi_h=0, roi_w=0) -> NccProblem:
    return NccProblem(mode=mode, score=score, subpix=subpix, image_h=image_h, image_w=image_w,
                      image_pitch=image_w if image_pitch is None else image_pitch, tmpl_h=tmpl_h, tmpl_w=tmpl_w,
                      search_y=search_y, search_x=search_x, step_y=step_y, step_x=step_x, batch=batch,
                      shard_rank=shard_rank, shard_count=shard_count, flags=flags, n_templates=n_templates,
                      roi_h=roi_h, roi_w=roi_w)


# ---------------------------------------------------------------- C-ABI names
def ncc_plan_create(problem: NccProblem, device: int = 0) -> int:
    h = ctypes.c_void_p()
    _check(lib().ncc_plan_create(ctypes.byref(problem), int(device), ctypes.byref(h)), "ncc_plan_create")
    return h.value


def ncc_plan_destroy(plan) -> None:
    _check(lib().ncc_plan_destroy(plan), "ncc_plan_destroy")


def ncc_plan_query(plan) -> NccPlanInfo:
    info = NccPlanInfo()
    _check(lib().ncc_plan_query(plan, ctypes.byref(info), ctypes.sizeof(info)), "ncc_plan_query")
    return info


def ncc_plan_timing(plan) -> NccTiming:
    t = NccTiming()
    _check(lib().ncc_plan_timing(plan, ctypes.byref(t)), "ncc_plan_timing")
    return t


def ncc_match(plan, images, tmpl, tmpl_pitch, scores, peaks, stream) -> None:
    _check(lib().ncc_match(plan, _ptr(images), _ptr(tmpl), int(tmpl_pitch), _ptr(scores), _ptr(peaks), stream),
           "ncc_match")


def ncc_match_rois(plan, images, tmpls, tmpl_pitch, rois, scores, peaks, stream) -> None:
    _check(lib().ncc_match_rois(plan, _ptr(images), _ptr(tmpls), int(tmpl_pitch), _ptr(rois), _ptr(scores),
                                _ptr(peaks), stream), "ncc_match_rois")


def piv_correlate(plan, frames_a, frames_b, vectors, stream) -> None:
    _check(lib().piv_correlate(plan, _ptr(frames_a), _ptr(frames_b), _ptr(vectors), stream), "piv_correlate")


def piv_correlate_ex(plan, frames_a, frames_b, scores, vectors, stream) -> None:
    _check(lib().piv_correlate_ex(plan, _ptr(frames_a), _ptr(frames_b), _ptr(scores), _ptr(vectors), stream),
           "piv_correlate_ex")


def ncc_match_host(plan, h_images, h_tmpl, tmpl_pitch, h_scores, h_peaks, stream) -> None:
    _check(lib().ncc_match_host(plan, _ptr(h_images), _ptr(h_tmpl), int(tmpl_pitch), _ptr(h_scores),
                                _ptr(h_peaks), stream), "ncc_match_host")


def piv_correlate_host(plan, h_a, h_b, h_vectors, stream) -> None:
    _check(lib().piv_correlate_host(plan, _ptr(h_a), _ptr(h_b), _ptr(h_vectors), stream), "piv_correlate_host")


def ncc_status_string(s: int) -> str:
    return lib().ncc_status_string(int(s)).decode()


def ncc_specialize(problem: NccProblem) -> tuple[str, bool]:
    """Compile (or find) the specialised kernel for `problem` into the binary cache (no GPU)."""
    buf = ctypes.create_string_buffer(96)
    now = ctypes.c_int32(0)
    _check(lib().ncc_specialize(ctypes.byref(problem), buf, 96, ctypes.byref(now)), "ncc_specialize")
    return buf.value.decode(), bool(now.value)
