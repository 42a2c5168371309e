"""Python-side names of the C ABI (include/mg.h): marshalling only, no arithmetic."""
from __future__ import annotations

import ctypes as C

import numpy as np

from . import _lib
from ._lib import check, load, mg_plan_info, mg_plan_opts, mg_profile, mg_tensor


def _i32(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.int32))


def _ptr_i32(a: np.ndarray):
    return a.ctypes.data_as(C.POINTER(C.c_int32)) if a.size else None


class Plan:
    """mg_plan_create / mg_plan_create_ex (metadata built once before inference).

    Args follow include/mg.h: L, heads, d, window, global_idx (int array), extra_idx (int [n, 2]).
    Options (test/ablation): block, force_all_fine, strip_max_cols, num_sms, fine_kernel
    (0 = warp-level tensor-core CSR kernel, 1 = CUDA-core CSR kernel), concurrency (0 = default,
    1 = serial fine -> coarse, 2 = concurrent streams with last-finisher row merge, 3 = SM split:
    coarse kernel on a share of the SMs, fine kernel beside it with dynamic rows), tau (tile
    density threshold; 0 = band rule), dense_chunk (column tiles per dense-row item; 0 = default 8,
    -1 = no split).
    """

    def __init__(self, L: int, heads: int, d: int, window: int, global_idx=(), extra_idx=None, *,
                 block: int = 0, force_all_fine: bool = False, strip_max_cols: int = 0, num_sms: int = 0,
                 fine_kernel: int = 0, concurrency: int = 0, tau: float = 0.0, dense_chunk: int = 0):
        lib = load()
        g = _i32(list(global_idx) if not isinstance(global_idx, np.ndarray) else global_idx).reshape(-1)
        e = _i32(np.zeros((0, 2)) if extra_idx is None else extra_idx).reshape(-1, 2)
        self._handle = C.c_void_p()
        self._lib = lib
        opts = mg_plan_opts(block, int(force_all_fine), strip_max_cols, num_sms, fine_kernel, concurrency, tau,
                            dense_chunk)
        if block or force_all_fine or strip_max_cols or num_sms or fine_kernel or concurrency or tau or dense_chunk:
            st = lib.mg_plan_create_ex(L, heads, d, window, _ptr_i32(g), g.size, _ptr_i32(e), e.shape[0],
                                       C.byref(opts), C.byref(self._handle))
        else:
            st = lib.mg_plan_create(L, heads, d, window, _ptr_i32(g), g.size, _ptr_i32(e), e.shape[0],
                                    C.byref(self._handle))
        check(st)
        self.L, self.heads, self.d, self.window = L, heads, d, window

    @property
    def handle(self):
        return self._handle

    def info(self) -> dict:
        inf = mg_plan_info()
        check(self._lib.mg_plan_info_get(self._handle, C.byref(inf)))
        return {name: getattr(inf, name) for name, _ in mg_plan_info._fields_ if name != "reserved"}

    def export(self) -> dict:
        inf = self.info()
        b = inf["block"]
        wpr = -(-b // 64)
        out = {
            "bsr_row_ptr": np.zeros(inf["n_row_blocks"] + 1, np.int32),
            "bsr_col": np.zeros(inf["n_tiles"], np.int32),
            "tile_masks": np.zeros((inf["n_tiles"], b, wpr), np.uint64),
            "csr_row_ptr": np.zeros(inf["L"] + 1, np.int32),
            "csr_col": np.zeros(inf["nnz_fine"], np.int32),
            "global_rows": np.zeros(inf["n_global"], np.int32),
        }
        i32 = lambda a: a.ctypes.data_as(C.POINTER(C.c_int32))
        check(self._lib.mg_plan_export(self._handle, i32(out["bsr_row_ptr"]), i32(out["bsr_col"]),
                                       out["tile_masks"].ctypes.data_as(C.POINTER(C.c_uint64)),
                                       i32(out["csr_row_ptr"]), i32(out["csr_col"]), i32(out["global_rows"])))
        return out

    def set_profiling(self, enable: bool = True) -> None:
        """mg_plan_set_profiling: record CUDA events around each kernel of every forward."""
        check(self._lib.mg_plan_set_profiling(self._handle, int(enable)))

    def get_profile(self) -> dict:
        """mg_plan_get_profile: summed per-kernel-class device ms since the last reset (then resets)."""
        pr = mg_profile()
        check(self._lib.mg_plan_get_profile(self._handle, C.byref(pr)))
        return {"calls": pr.calls, "fine_ms": pr.fine_ms, "coarse_ms": pr.coarse_ms, "total_ms": pr.total_ms}

    def get_profile_calls(self) -> tuple[dict, list]:
        """mg_plan_get_profile_calls: as get_profile, plus each call's first-to-last-launch ms."""
        pr = mg_profile()
        cap = 1 << 16
        buf = (C.c_double * cap)()
        check(self._lib.mg_plan_get_profile_calls(self._handle, C.byref(pr), buf, cap))
        per = [buf[i] for i in range(min(pr.calls, cap))]
        return {"calls": pr.calls, "fine_ms": pr.fine_ms, "coarse_ms": pr.coarse_ms, "total_ms": pr.total_ms}, per

    def set_trace(self, buf=None) -> None:
        """mg_plan_set_trace: zeroed device int64 tensor of >= 128 elements (MG_TRACE builds add their
        per-role phase counters to it, see tools/trace_coarse.py) or None to stop."""
        if buf is None:
            check(self._lib.mg_plan_set_trace(self._handle, None, 0))
        else:
            check(self._lib.mg_plan_set_trace(self._handle, C.c_void_p(buf.data_ptr()), buf.numel()))

    def close(self):
        if getattr(self, "_handle", None) is not None and self._handle.value:
            self._lib.mg_plan_destroy(self._handle)
            self._handle = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def autotune_plan(L: int, heads: int, d: int, window: int, global_idx, extra_idx, Q, K, V, O=None, stream=None):
    """mg_plan_autotune: the fastest of the block {128, 64} x tau {0, 0.1, 0.25, 0.5} plans of this
    pattern, timed on the given device tensors (O is scratch). Returns (plan, chosen options, ms)."""
    import torch
    lib = load()
    g = _i32(list(global_idx) if not isinstance(global_idx, np.ndarray) else global_idx).reshape(-1)
    e = _i32(np.zeros((0, 2)) if extra_idx is None else extra_idx).reshape(-1, 2)
    if O is None:
        O = torch.empty(Q.shape, dtype=Q.dtype, device=Q.device)
    dq, dk, dv, do = tensor_desc(Q), tensor_desc(K), tensor_desc(V), tensor_desc(O)
    h = C.c_void_p()
    chosen = mg_plan_opts()
    ms = C.c_double()
    check(lib.mg_plan_autotune(L, heads, d, window, _ptr_i32(g), g.size, _ptr_i32(e), e.shape[0], C.byref(dq),
                               C.byref(dk), C.byref(dv), C.byref(do), _stream_ptr(stream), C.byref(h),
                               C.byref(chosen), C.byref(ms)))
    plan = Plan.__new__(Plan)
    plan._handle, plan._lib = h, lib
    plan.L, plan.heads, plan.d, plan.window = L, heads, d, window
    return plan, {"block": chosen.block, "tau": chosen.tau}, ms.value


class BatchedPlan(Plan):
    """mg_plan_create_batched: one plan for a batch whose samples have their own global tokens and
    extra pairs (lists of arrays, one per sample). Same options as Plan."""

    def __init__(self, L: int, heads: int, d: int, window: int, global_idx_per_sample, extra_idx_per_sample=None,
                 **opts):
        lib = load()
        B = len(global_idx_per_sample)
        extras = extra_idx_per_sample if extra_idx_per_sample is not None else [None] * B
        if len(extras) != B:
            raise ValueError("one extra_idx array per sample")
        gl = [_i32(np.asarray(g, dtype=np.int64)).reshape(-1) for g in global_idx_per_sample]
        ex = [_i32(np.zeros((0, 2)) if e is None else e).reshape(-1, 2) for e in extras]
        gptr = np.zeros(B + 1, np.int64)
        eptr = np.zeros(B + 1, np.int64)
        gptr[1:] = np.cumsum([g.size for g in gl])
        eptr[1:] = np.cumsum([e.shape[0] for e in ex])
        g_all = _i32(np.concatenate(gl) if B else np.zeros(0))
        e_all = _i32(np.concatenate(ex) if B else np.zeros((0, 2))).reshape(-1, 2)
        self._handle = C.c_void_p()
        self._lib = lib
        o = mg_plan_opts(opts.get("block", 0), int(opts.get("force_all_fine", False)), opts.get("strip_max_cols", 0),
                         opts.get("num_sms", 0), opts.get("fine_kernel", 0), opts.get("concurrency", 0),
                         opts.get("tau", 0.0), opts.get("dense_chunk", 0))
        i64p = lambda a: a.ctypes.data_as(C.POINTER(C.c_int64))
        check(lib.mg_plan_create_batched(L, heads, d, window, B, i64p(gptr), _ptr_i32(g_all), i64p(eptr),
                                         _ptr_i32(e_all), C.byref(o), C.byref(self._handle)))
        self.L, self.heads, self.d, self.window, self.batch = L, heads, d, window, B


def tensor_desc(t) -> mg_tensor:
    """mg_tensor for a torch tensor viewed as [B, H, L, d] (any strides with a unit d-stride)."""
    import torch
    if t.dim() != 4:
        raise ValueError("expected a 4-D [B, H, L, d] tensor")
    if t.dtype == torch.bfloat16:
        dt = _lib.MG_BF16
    elif t.dtype == torch.float16:
        dt = _lib.MG_FP16
    else:
        raise TypeError(f"unsupported dtype {t.dtype}")
    if t.stride(3) != 1:
        raise ValueError("head_dim stride must be 1")
    B, H, L, d = t.shape
    sb, sh, sl, _ = t.stride()
    return mg_tensor(t.data_ptr(), dt, 0, B, H, L, d, sb, sh, sl)


def _stream_ptr(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return C.c_void_p(stream.cuda_stream)


def sparse_attention_fwd(plan: Plan, Q, K, V, O=None, stream=None):
    """mg_sparse_attention_fwd on device tensors [B, H, L, d]; returns O (allocated if None)."""
    import torch
    if O is None:
        O = torch.empty(Q.shape, dtype=Q.dtype, device=Q.device)
    dq, dk, dv, do = tensor_desc(Q), tensor_desc(K), tensor_desc(V), tensor_desc(O)
    check(plan._lib.mg_sparse_attention_fwd(plan.handle, C.byref(dq), C.byref(dk), C.byref(dv), C.byref(do),
                                            _stream_ptr(stream)))
    return O


def sparse_attention_fwd_padded(plan: Plan, Q, K, V, valid_len, O=None, stream=None):
    """mg_sparse_attention_fwd_padded: valid_len is a device int32 tensor [B] (tokens >= valid_len[b]
    are padding: masked as columns, zero output rows)."""
    import torch
    if O is None:
        O = torch.empty(Q.shape, dtype=Q.dtype, device=Q.device)
    if valid_len.dtype != torch.int32 or not valid_len.is_cuda or valid_len.numel() != Q.shape[0]:
        raise ValueError("valid_len must be a CUDA int32 tensor with one entry per batch element")
    dq, dk, dv, do = tensor_desc(Q), tensor_desc(K), tensor_desc(V), tensor_desc(O)
    check(plan._lib.mg_sparse_attention_fwd_padded(plan.handle, C.byref(dq), C.byref(dk), C.byref(dv), C.byref(do),
                                                   C.c_void_p(valid_len.data_ptr()), _stream_ptr(stream)))
    return O


def sparse_attention_fwd_host(plan: Plan, Q, K, V, O, stream=None):
    """mg_sparse_attention_fwd_host on dense HOST tensors (pinned for async copies). Asynchronous:
    synchronise `stream` before reading O."""
    dq, dk, dv, do = tensor_desc(Q), tensor_desc(K), tensor_desc(V), tensor_desc(O)
    check(plan._lib.mg_sparse_attention_fwd_host(plan.handle, C.byref(dq), C.byref(dk), C.byref(dv),
                                                 C.byref(do), _stream_ptr(stream)))
    return O


def staged_sizes(plan: Plan) -> dict:
    """mg_staged_get_sizes: per-(batch, head) element counts of the staged buffers."""
    z = _lib.mg_staged_sizes()
    check(plan._lib.mg_staged_get_sizes(plan.handle, C.byref(z)))
    return {name: getattr(z, name) for name, _ in z._fields_}


def _ptr(t):
    return None if t is None or t.numel() == 0 else C.c_void_p(t.data_ptr())


def staged_buffers(plan: Plan, batch: int, dtype, device="cuda") -> dict:
    """Allocate the staged-mode buffers (S fp32, P in `dtype`, O_csr fp32) for `batch`."""
    import torch
    z = staged_sizes(plan)
    BH = batch * plan.heads
    f32 = dict(dtype=torch.float32, device=device)
    return {"S_tiles": torch.empty(BH, z["tile_elems"], **f32), "S_csr": torch.empty(BH, z["csr_elems"], **f32),
            "S_global": torch.empty(BH, z["global_elems"], **f32),
            "P_tiles": torch.empty(BH, z["tile_elems"], dtype=dtype, device=device),
            "P_csr": torch.empty(BH, z["csr_elems"], dtype=dtype, device=device),
            "P_global": torch.empty(BH, z["global_elems"], dtype=dtype, device=device),
            "O_csr": torch.empty(BH, z["ocsr_elems"], **f32), "lpad": z["lpad"]}


def staged_sddmm(plan: Plan, Q, K, bufs: dict, stream=None):
    """mg_staged_sddmm: coarse, fine and dense-row scores into bufs S_tiles / S_csr / S_global."""
    dq, dk = tensor_desc(Q), tensor_desc(K)
    check(plan._lib.mg_staged_sddmm(plan.handle, C.byref(dq), C.byref(dk), _ptr(bufs["S_tiles"]),
                                    _ptr(bufs["S_csr"]), _ptr(bufs["S_global"]), _stream_ptr(stream)))


def staged_softmax(plan: Plan, batch: int, bufs: dict, stream=None):
    """mg_staged_softmax: compound SpSoftmax of the S buffers into the P buffers."""
    import torch
    dt = _lib.MG_BF16 if bufs["P_tiles"].dtype == torch.bfloat16 else _lib.MG_FP16
    check(plan._lib.mg_staged_softmax(plan.handle, batch, dt, _ptr(bufs["S_tiles"]), _ptr(bufs["S_csr"]),
                                      _ptr(bufs["S_global"]), _ptr(bufs["P_tiles"]), _ptr(bufs["P_csr"]),
                                      _ptr(bufs["P_global"]), _stream_ptr(stream)))


def staged_spmm(plan: Plan, V, O, bufs: dict, stream=None):
    """mg_staged_spmm: O = P V over the tiles, the CSR part (via O_csr) and the dense rows."""
    dv, do = tensor_desc(V), tensor_desc(O)
    check(plan._lib.mg_staged_spmm(plan.handle, _ptr(bufs["P_tiles"]), _ptr(bufs["P_csr"]), _ptr(bufs["P_global"]),
                                   C.byref(dv), C.byref(do), _ptr(bufs["O_csr"]), _stream_ptr(stream)))
    return O


def sparse_attention_fwd_staged(plan: Plan, Q, K, V, O=None, stream=None, multi_stream: bool = False):
    """mg_sparse_attention_fwd_staged(_ex): the paper's dataflow (SDDMM -> SpSoftmax -> SpMM kernels);
    multi_stream=True runs each step's coarse and fine kernels on two streams."""
    import torch
    if O is None:
        O = torch.empty(Q.shape, dtype=Q.dtype, device=Q.device)
    dq, dk, dv, do = tensor_desc(Q), tensor_desc(K), tensor_desc(V), tensor_desc(O)
    check(plan._lib.mg_sparse_attention_fwd_staged_ex(plan.handle, C.byref(dq), C.byref(dk), C.byref(dv),
                                                      C.byref(do), 1 if multi_stream else 0, _stream_ptr(stream)))
    return O


def selftest_umma(mode: int, A, B, D, stream=None):
    """mg_selftest_umma: one tcgen05 MMA on device buffers (diagnostics)."""
    check(load().mg_selftest_umma(mode, C.c_void_p(A.data_ptr()), C.c_void_p(B.data_ptr()),
                                  C.c_void_p(D.data_ptr()), _stream_ptr(stream)))
    return D
