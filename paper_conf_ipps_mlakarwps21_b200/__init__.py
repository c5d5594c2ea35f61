"""B200-native batch-based Reverse Cuthill-McKee (Mlakar et al., IPDPS'21).

Thin ctypes binding over ``librcm.so`` (the C ABI declared in
``include/rcm.h``).  Functions keep the C names; this module only marshals
arguments (torch CUDA tensors -> device pointers, the current CUDA stream).
Every step of the hot path runs in the library's CUDA kernels; there is no
CPU fallback: importing this package fails loudly when the extension is
missing.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# RCM_LIB: an alternative in-tree build of the same library (A/B experiments, tools/)
LIB_PATH = os.environ.get("RCM_LIB") or os.path.join(_HERE, "librcm.so")

RCM_START_FIXED = 0
RCM_START_MIN_DEGREE = 1
RCM_START_PSEUDO_PERIPHERAL = 2

RCM_FLAG_NO_OVERHANG = 0x1
RCM_FLAG_NO_EARLY = 0x2
RCM_FLAG_NO_SORT = 0x4
RCM_FLAG_FORCE_CHAIN = 0x8
RCM_FLAG_SERIAL_CHAIN = 0x10
RCM_FLAG_LEVELED = 0x20
RCM_FLAG_MULTI_BATCH = 0x40
RCM_FLAG_BATCHED_ONLY = 0x80

STATUS = {
    0: "RCM_OK", 1: "RCM_ERR_INVALID_ARGUMENT", 2: "RCM_ERR_BAD_CSR", 3: "RCM_ERR_NOT_SYMMETRIC",
    4: "RCM_ERR_OUT_OF_MEMORY", 5: "RCM_ERR_CAPACITY", 6: "RCM_ERR_HANG", 7: "RCM_ERR_CUDA",
    8: "RCM_ERR_NCCL",
}

# every symbol include/rcm.h declares
EXPORTS = ["rcm_default_options", "rcm_plan_create", "rcm_reorder", "rcm_reorder_batched",
           "rcm_find_pseudo_peripheral", "rcm_sync_status", "rcm_get_stats", "rcm_get_timing", "rcm_plan_info",
           "rcm_plan_destroy", "rcm_status_string", "rcm_probe_hop", "rcm_reorder_batched_host"]


class rcm_options_t(ctypes.Structure):
    _fields_ = [("batch_nodes", ctypes.c_int32), ("temp_elems", ctypes.c_int32),
                ("blocks_per_sm", ctypes.c_int32), ("validate", ctypes.c_int32),
                ("collect_stats", ctypes.c_int32), ("queue_capacity", ctypes.c_int32),
                ("solo_threshold", ctypes.c_int32), ("flags", ctypes.c_int32)]


STAGES = ("dequeue", "parents", "discover", "wait_discovered", "rediscover_count", "sort",
          "wait_counted", "output", "generate", "other")


class rcm_stats_t(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int64) for n in (
        "batches_generated", "batches_dequeued", "batches_executed", "batches_empty",
        "rediscover_early", "rediscover_late", "candidates_speculative", "candidates_removed",
        "oversize_batches", "components", "overhang_forwards", "solo_problems")] + [
        ("stage_cycles", ctypes.c_int64 * 10)]

    def as_dict(self):
        d = {n: int(getattr(self, n)) for n, _ in self._fields_ if n != "stage_cycles"}
        cyc = [int(x) for x in self.stage_cycles]
        if any(cyc):
            d["stage_cycles"] = dict(zip(STAGES, cyc))
        return d


class RCMError(RuntimeError):
    def __init__(self, status: int, where: str = ""):
        self.status = status
        super().__init__(f"{where}: {STATUS.get(status, status)}")


_lib = None


def _load():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"librcm.so not built ({LIB_PATH}); run __graft_entry__.build() or "
                          "python paper_conf_ipps_mlakarwps21_b200/build.py")
    lib = ctypes.CDLL(LIB_PATH)
    vp, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
    lib.rcm_default_options.argtypes = [ctypes.POINTER(rcm_options_t)]
    lib.rcm_default_options.restype = None
    lib.rcm_plan_create.argtypes = [ctypes.POINTER(vp), i64, i64, ctypes.POINTER(rcm_options_t)]
    lib.rcm_reorder.argtypes = [vp, i32, i64, vp, vp, i32, i32, vp, vp, vp]
    lib.rcm_reorder_batched.argtypes = [vp, i32, i64, i64, vp, vp, vp, vp, i32, vp, vp, vp]
    lib.rcm_find_pseudo_peripheral.argtypes = [vp, i32, i64, vp, vp, i32, vp, vp]
    lib.rcm_sync_status.argtypes = [vp, vp]
    lib.rcm_get_stats.argtypes = [vp, ctypes.POINTER(rcm_stats_t)]
    lib.rcm_plan_info.argtypes = [vp, ctypes.POINTER(ctypes.c_int64)]
    lib.rcm_get_timing.argtypes = [vp, ctypes.POINTER(ctypes.c_double)]
    lib.rcm_plan_destroy.argtypes = [vp]
    lib.rcm_plan_destroy.restype = None
    lib.rcm_reorder_batched_host.argtypes = [vp, i32, vp, vp, vp, vp, i32, vp, vp, vp, vp, vp, vp, vp, vp, i32, vp]
    lib.rcm_reorder_batched_host.restype = i32
    lib.rcm_probe_hop.argtypes = [i32, i32, i32, ctypes.POINTER(ctypes.c_double)]
    lib.rcm_probe_hop.restype = i32
    lib.rcm_status_string.argtypes = [i32]
    lib.rcm_status_string.restype = ctypes.c_char_p
    for f in ("rcm_plan_create", "rcm_reorder", "rcm_reorder_batched", "rcm_find_pseudo_peripheral",
              "rcm_sync_status", "rcm_get_stats", "rcm_get_timing", "rcm_plan_info"):
        getattr(lib, f).restype = i32
    _lib = lib
    return lib


_load()


# ------------------------------------------------------------ marshalling
def _ptr(t, dtype=None, name="tensor"):
    if t is None:
        return None
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA tensor")
    if dtype is not None and t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    return ctypes.c_void_p(t.data_ptr())


def _stream(stream):
    if stream is None:
        import torch
        return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return ctypes.c_void_p(stream)
    return ctypes.c_void_p(stream.cuda_stream)


def _check(st, where):
    if st != 0:
        raise RCMError(st, where)


def rcm_default_options(**kw) -> rcm_options_t:
    o = rcm_options_t()
    _load().rcm_default_options(ctypes.byref(o))
    for k, v in kw.items():
        setattr(o, k, int(v))
    return o


def rcm_plan_create(n_max: int, nnz_max: int, options: rcm_options_t | None = None):
    """Returns an opaque plan handle (ctypes.c_void_p)."""
    h = ctypes.c_void_p()
    st = _load().rcm_plan_create(ctypes.byref(h), int(n_max), int(nnz_max),
                                 ctypes.byref(options) if options is not None else None)
    _check(st, "rcm_plan_create")
    return h


def rcm_reorder(plan, n: int, nnz: int, row_ptr, col_idx, mode: int, start: int, perm,
                iperm=None, stream=None) -> None:
    import torch
    st = _load().rcm_reorder(plan, int(n), int(nnz), _ptr(row_ptr, torch.int32, "row_ptr"),
                             _ptr(col_idx, torch.int32, "col_idx"), int(mode), int(start),
                             _ptr(perm, torch.int32, "perm"), _ptr(iperm, torch.int32, "iperm"),
                             _stream(stream))
    _check(st, "rcm_reorder")


def rcm_reorder_batched(plan, num_mats: int, total_nodes: int, total_nnz: int, node_off, nnz_off,
                        row_ptr_local, col_idx_local, mode: int, starts, perm_local, stream=None) -> None:
    import torch
    st = _load().rcm_reorder_batched(
        plan, int(num_mats), int(total_nodes), int(total_nnz), _ptr(node_off, torch.int64, "node_off"),
        _ptr(nnz_off, torch.int64, "nnz_off"), _ptr(row_ptr_local, torch.int32, "row_ptr_local"),
        _ptr(col_idx_local, torch.int32, "col_idx_local"), int(mode), _ptr(starts, torch.int32, "starts"),
        _ptr(perm_local, torch.int32, "perm_local"), _stream(stream))
    _check(st, "rcm_reorder_batched")


def _hptr(t, dtype, name):
    """Host pointer of a CPU tensor (pinned for full PCIe bandwidth)."""
    import torch
    if t is None:
        return None
    if not isinstance(t, torch.Tensor) or t.is_cuda:
        raise TypeError(f"{name} must be a CPU tensor")
    if t.dtype != dtype or not t.is_contiguous():
        raise TypeError(f"{name} must be a contiguous {dtype} tensor")
    return ctypes.c_void_p(t.data_ptr())


def rcm_reorder_batched_host(plan, num_mats: int, node_off_h, nnz_off_h, row_ptr_h, col_idx_h, mode: int,
                             starts_h, perm_h, node_off_d, nnz_off_d, row_ptr_d, col_idx_d, starts_d, perm_d,
                             chunks: int = 8, stream=None) -> None:
    import torch
    st = _load().rcm_reorder_batched_host(
        plan, int(num_mats), _hptr(node_off_h, torch.int64, "node_off_h"), _hptr(nnz_off_h, torch.int64, "nnz_off_h"),
        _hptr(row_ptr_h, torch.int32, "row_ptr_h"), _hptr(col_idx_h, torch.int32, "col_idx_h"), int(mode),
        _hptr(starts_h, torch.int32, "starts_h"), _hptr(perm_h, torch.int32, "perm_h"),
        _ptr(node_off_d, torch.int64, "node_off_d"), _ptr(nnz_off_d, torch.int64, "nnz_off_d"),
        _ptr(row_ptr_d, torch.int32, "row_ptr_d"), _ptr(col_idx_d, torch.int32, "col_idx_d"),
        _ptr(starts_d, torch.int32, "starts_d"), _ptr(perm_d, torch.int32, "perm_d"), int(chunks), _stream(stream))
    _check(st, "rcm_reorder_batched_host")


def rcm_find_pseudo_peripheral(plan, n: int, nnz: int, row_ptr, col_idx, start: int, out, stream=None):
    import torch
    st = _load().rcm_find_pseudo_peripheral(plan, int(n), int(nnz), _ptr(row_ptr, torch.int32, "row_ptr"),
                                            _ptr(col_idx, torch.int32, "col_idx"), int(start),
                                            _ptr(out, torch.int32, "out"), _stream(stream))
    _check(st, "rcm_find_pseudo_peripheral")


def rcm_sync_status(plan, stream=None) -> int:
    return int(_load().rcm_sync_status(plan, _stream(stream)))


def rcm_get_stats(plan) -> dict:
    s = rcm_stats_t()
    _check(_load().rcm_get_stats(plan, ctypes.byref(s)), "rcm_get_stats")
    return s.as_dict()


def rcm_get_timing(plan) -> dict:
    a = (ctypes.c_double * 7)()
    _check(_load().rcm_get_timing(plan, a), "rcm_get_timing")
    return dict(zip(("prologue_ms", "setup_ms", "traversal_ms", "components_ms", "total_ms",
                     "cc_label_ms", "cc_sort_layout_ms"),
                    [float(x) for x in a]))


def rcm_plan_info(plan) -> dict:
    a = (ctypes.c_int64 * 8)()
    _check(_load().rcm_plan_info(plan, a), "rcm_plan_info")
    return dict(zip(("blocks", "threads", "batch_nodes", "temp_elems", "smem_bytes", "queue_slots",
                     "solo_blocks", "solo_smem_bytes"), [int(x) for x in a]))


def rcm_plan_destroy(plan) -> None:
    if plan:
        _load().rcm_plan_destroy(plan)


def rcm_probe_hop(sm_a: int, sm_b: int, iters: int = 2000) -> float:
    """One-way block-to-block hand-off time (ns) between SMs sm_a and sm_b."""
    out = ctypes.c_double()
    _check(_load().rcm_probe_hop(int(sm_a), int(sm_b), int(iters), ctypes.byref(out)), "rcm_probe_hop")
    return float(out.value)


def rcm_status_string(st: int) -> str:
    return _load().rcm_status_string(int(st)).decode()


# ------------------------------------------------------- convenience wrapper
class Plan:
    """Owns a plan; ``reorder`` allocates the output, runs, syncs, raises."""

    def __init__(self, n_max: int, nnz_max: int, **options):
        self.options = rcm_default_options(**options)
        self.handle = rcm_plan_create(n_max, nnz_max, self.options)

    def close(self):
        if self.handle:
            rcm_plan_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def info(self):
        return rcm_plan_info(self.handle)

    def stats(self):
        return rcm_get_stats(self.handle)

    def timing(self):
        return rcm_get_timing(self.handle)

    def reorder(self, row_ptr, col_idx, mode=RCM_START_MIN_DEGREE, start=0, perm=None, iperm=None,
                stream=None, sync=True):
        import torch
        n = row_ptr.numel() - 1
        nnz = col_idx.numel()
        if perm is None:
            perm = torch.empty(n, dtype=torch.int32, device=row_ptr.device)
        rcm_reorder(self.handle, n, nnz, row_ptr, col_idx, mode, start, perm, iperm, stream)
        if sync:
            _check(rcm_sync_status(self.handle, stream), "rcm_reorder (device)")
        return perm

    def reorder_batched(self, node_off, nnz_off, row_ptr_local, col_idx_local, total_nodes, total_nnz,
                        mode=RCM_START_MIN_DEGREE, starts=None, perm_local=None, stream=None, sync=True):
        import torch
        num = node_off.numel() - 1
        if perm_local is None:
            perm_local = torch.empty(total_nodes, dtype=torch.int32, device=row_ptr_local.device)
        rcm_reorder_batched(self.handle, num, total_nodes, total_nnz, node_off, nnz_off, row_ptr_local,
                            col_idx_local, mode, starts, perm_local, stream)
        if sync:
            _check(rcm_sync_status(self.handle, stream), "rcm_reorder_batched (device)")
        return perm_local

    def find_pseudo_peripheral(self, row_ptr, col_idx, start, stream=None):
        import torch
        out = torch.empty(1, dtype=torch.int32, device=row_ptr.device)
        rcm_find_pseudo_peripheral(self.handle, row_ptr.numel() - 1, col_idx.numel(), row_ptr, col_idx,
                                   start, out, stream)
        _check(rcm_sync_status(self.handle, stream), "rcm_find_pseudo_peripheral (device)")
        return int(out.item())
