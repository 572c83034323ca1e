"""Thin ctypes binding of libvpps.so (include/vpps.h) — argument marshalling only.

Every step of the hot path runs in the CUDA library; this module converts Python graphs to the
CSR `vpps_batch`, passes torch device pointers and the current CUDA stream, and turns status codes
into exceptions.  There is no CPU fallback: if libvpps.so is missing, importing raises.
"""
from __future__ import annotations

import ctypes as ct
import itertools
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libvpps.so")

CELLS = {"lstm": 0, "binary": 1, "childsum": 2, "bilstm": 3, "gru": 4, "rvnn": 5, "tdrnn": 6, "tdlstm": 7,
         "bilstmchar": 8}
STATUS = {0: "OK", -1: "INVALID", -2: "NOFIT", -3: "CUDA", -4: "GRAPH", -5: "STATE", -6: "NOMEM"}


class VppsError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"VPPS_E_{STATUS.get(status, status)}: {msg}")
        self.status = status


class _Shape(ct.Structure):
    _fields_ = [("rows", ct.c_int32), ("cols", ct.c_int32)]


class _Opset(ct.Structure):
    _fields_ = [("cell", ct.c_int32), ("E", ct.c_int32), ("H", ct.c_int32), ("C", ct.c_int32), ("mlp", ct.c_int32)]


_ALLOC_FN = ct.CFUNCTYPE(ct.c_void_p, ct.c_size_t, ct.c_void_p, ct.c_void_p)
_FREE_FN = ct.CFUNCTYPE(None, ct.c_void_p, ct.c_void_p, ct.c_void_p)


class _Options(ct.Structure):
    _fields_ = [("n_sm", ct.c_int32), ("ctas_per_sm", ct.c_int32), ("groups", ct.c_int32),
                ("device", ct.c_int32), ("plan_only", ct.c_int32), ("cluster", ct.c_int32),
                ("dataflow", ct.c_int32), ("level", ct.c_int32), ("chain", ct.c_int32),
                ("alloc", _ALLOC_FN), ("free", _FREE_FN), ("alloc_ctx", ct.c_void_p)]


def _torch_allocator(device: int):
    """vpps_alloc_fn / vpps_free_fn over torch's caching allocator (include/vpps.h): PyTorch supplies the
    library's device memory (north_star).  Returns the two ctypes callbacks (keep them alive)."""
    import torch

    def alloc(nbytes, stream, _ctx):
        try:
            return torch.cuda.caching_allocator_alloc(int(nbytes), device, stream or 0)
        except Exception:            # out of memory -> NULL -> VPPS_E_NOMEM
            return None

    def free(ptr, _stream, _ctx):
        try:
            torch.cuda.caching_allocator_delete(ptr)
        except Exception:            # interpreter shutdown: torch already torn down
            pass
    return _ALLOC_FN(alloc), _FREE_FN(free)


class _Batch(ct.Structure):
    _fields_ = [("n_graphs", ct.c_int32), ("graph_ptr", ct.c_void_p), ("child_ptr", ct.c_void_p),
                ("children", ct.c_void_p), ("token", ct.c_void_p), ("label", ct.c_void_p),
                ("char_ptr", ct.c_void_p), ("chars", ct.c_void_p)]


class _Info(ct.Structure):
    _fields_ = [("n_words", ct.c_int64), ("pool_words", ct.c_int64), ("zero_words", ct.c_int64),
                ("loss_word", ct.c_int64), ("n_barriers", ct.c_int32), ("n_levels", ct.c_int32),
                ("n_nodes", ct.c_int64), ("n_heads", ct.c_int64), ("flops", ct.c_double),
                ("act_bytes", ct.c_double), ("blob_words", ct.c_int64), ("kernel_flops", ct.c_double)]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'` "
                          "(the VPPS path has no CPU fallback)")
    lib = ct.CDLL(LIB_PATH)
    P, I32, I64, F, VP = ct.POINTER, ct.c_int32, ct.c_int64, ct.c_float, ct.c_void_p
    sig = {
        "vpps_define_model": [P(_Shape), I32, P(_Opset), P(_Options), P(VP)],
        "vpps_layout": [VP, P(I64), P(I64)],
        "vpps_bind_buffers": [VP, VP, VP],
        "vpps_partition_table": [VP, P(P(I32)), P(I64)],
        "vpps_plan_info": [VP, P(I32), P(I32), P(I32), P(I32)],
        "vpps_paper_deal": [P(_Shape), I32, I32, I32, I32, I32, I32, VP, P(I64), P(I64)],
        "vpps_paper_choose_cps": [P(_Shape), I32, I32, I32, I32, I32],
        "vpps_build_script": [VP, P(_Batch), P(VP)],
        "vpps_script_words": [VP, P(P(ct.c_uint32)), P(I64)],
        "vpps_script_blob": [VP, P(P(ct.c_uint32)), P(I64), P(I64), P(I64)],
        "vpps_script_info_get": [VP, P(_Info)],
        "vpps_upload_script": [VP, VP],
        "vpps_fwd_bwd": [VP, VP, VP, I64, VP, VP],
        "vpps_fwd_bwd_sgd": [VP, VP, VP, I64, VP, F, F, VP],
        "vpps_sgd_step": [VP, F, F, VP],
        "vpps_get_stale_loss": [VP, P(F)],
        "vpps_sync_get_latest_loss": [VP, P(F)],
        "vpps_pool_ptr": [VP, P(VP), P(I64)],
        "vpps_set_timing_events": [VP, VP, VP],
        "vpps_set_kernel_events": [VP, VP, VP],
        "vpps_set_gemm_trace": [VP, VP],
        "vpps_set_profile_buffer": [VP, VP, I64],
        "vpps_destroy_script": [VP],
        "vpps_destroy_model": [VP],
        "vpps_last_error": [],
        "vpps_variants": [VP, I32],
    }
    sig["vpps_gemm_f32"] = [VP, I32, I32, I32, I32, I32, VP, I32, VP, I32, VP, I32, F]
    for name, args in sig.items():
        fn = getattr(lib, name)
        fn.argtypes = args
        fn.restype = ct.c_int32
    lib.vpps_last_error.restype = ct.c_char_p
    lib.vpps_destroy_script.restype = None
    lib.vpps_destroy_model.restype = None
    return lib


_lib = _load()


def _check(st: int):
    if st != 0:
        raise VppsError(st, _lib.vpps_last_error().decode())


def _stream_ptr(stream):
    if stream is None:
        import torch
        return ct.c_void_p(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return ct.c_void_p(stream)
    return ct.c_void_p(stream.cuda_stream)


def param_shapes(cell: str, H: int, E: int, C: int, mlp: int = 256, Ec: int = 64, Vc: int = 64):
    """Parameter order of vpps_define_model (include/vpps.h); bias shapes are (n,)."""
    if cell == "bilstmchar":
        Hc = E // 2
        return [("Wf", (4 * H, E)), ("Uf", (4 * H, H)), ("Wb", (4 * H, E)), ("Ub", (4 * H, H)),
                ("W_mlp", (mlp, 2 * H)), ("W_tag", (C, mlp)),
                ("C_emb", (Vc, Ec)), ("Wcf", (4 * Hc, Ec)), ("Ucf", (4 * Hc, Hc)), ("Wcb", (4 * Hc, Ec)),
                ("Ucb", (4 * Hc, Hc)),
                ("bf", (4 * H,)), ("bb", (4 * H,)), ("b_mlp", (mlp,)), ("b_tag", (C,)),
                ("bcf", (4 * Hc,)), ("bcb", (4 * Hc,))]
    if cell == "bilstm":
        return [("Wf", (4 * H, E)), ("Uf", (4 * H, H)), ("Wb", (4 * H, E)), ("Ub", (4 * H, H)),
                ("W_mlp", (mlp, 2 * H)), ("W_tag", (C, mlp)),
                ("bf", (4 * H,)), ("bb", (4 * H,)), ("b_mlp", (mlp,)), ("b_tag", (C,))]
    if cell == "lstm":
        return [("W", (4 * H, E)), ("U", (4 * H, H)), ("W_out", (C, H)), ("b", (4 * H,)), ("b_out", (C,))]
    if cell == "tdrnn":
        return [("W", (H, 2 * H)), ("W_out", (C, H)), ("b", (H,)), ("b_out", (C,))]
    if cell == "rvnn":
        return [("W_leaf", (H, E)), ("W_int", (H, 2 * H)), ("W_out", (C, H)), ("b_leaf", (H,)), ("b_int", (H,)),
                ("b_out", (C,))]
    if cell == "gru":
        return [("W", (3 * H, E)), ("U", (3 * H, H)), ("W_out", (C, H)), ("b_i", (3 * H,)), ("b_h", (3 * H,)),
                ("b_out", (C,))]
    if cell in ("binary", "tdlstm"):
        return [("W_iou", (3 * H, E)), ("U_iou", (3 * H, 2 * H)), ("U_fl", (H, H)), ("U_fr", (H, H)),
                ("W_out", (C, H)), ("b_iou", (3 * H,)), ("b_f", (H,)), ("b_out", (C,))]
    if cell == "childsum":
        return [("W_iou", (3 * H, E)), ("W_f", (H, E)), ("U_iou", (3 * H, H)), ("U_f", (H, H)),
                ("W_out", (C, H)), ("b_iou", (3 * H,)), ("b_f", (H,)), ("b_out", (C,))]
    raise ValueError(cell)


def gemm_f32(A, B, C, ta=False, tb=False, beta=0.0, M=None, N=None, K=None, lda=None, ldb=None, ldc=None,
             stream=None):
    """C = op(A) op(B) + beta C through vpps_gemm_f32 (include/vpps.h) on float32 CUDA tensors (row-major;
    leading dimensions default to the tensors' row strides)."""
    M = M if M is not None else C.shape[0]
    N = N if N is not None else C.shape[1]
    K = K if K is not None else (A.shape[0] if ta else A.shape[1])
    _check(_lib.vpps_gemm_f32(_stream_ptr(stream), int(ta), int(tb), M, N, K, ct.c_void_p(A.data_ptr()),
                              lda or A.stride(0), ct.c_void_p(B.data_ptr()), ldb or B.stride(0),
                              ct.c_void_p(C.data_ptr()), ldc or C.stride(0), beta))


def variants():
    buf = (ct.c_int32 * 256)()
    n = _lib.vpps_variants(ct.cast(buf, ct.c_void_p), 64)
    inv = {v: k for k, v in CELLS.items()}
    return [(inv[buf[4 * i]], buf[4 * i + 1], buf[4 * i + 2], buf[4 * i + 3]) for i in range(n)]


def paper_deal(mats, n_cta, tb, rpw, pack_rows=True, grads=False):
    """SPEC P0 dealer -> (rows int32 [n, 6] = matrix,row,cta,partition,warp,is_grad ; n_slots)."""
    sh = (_Shape * len(mats))(*[_Shape(r, c) for r, c in mats])
    n, slots = ct.c_int64(), ct.c_int64()
    _check(_lib.vpps_paper_deal(sh, len(mats), n_cta, tb, rpw, int(pack_rows), int(grads), None,
                                ct.byref(n), ct.byref(slots)))
    out = np.zeros((n.value, 6), dtype=np.int32)
    _check(_lib.vpps_paper_deal(sh, len(mats), n_cta, tb, rpw, int(pack_rows), int(grads),
                                out.ctypes.data_as(ct.c_void_p), ct.byref(n), ct.byref(slots)))
    return out, slots.value


def paper_choose_cps(mats, n_sm, tb=256, rpw=1, pack_rows=True):
    sh = (_Shape * len(mats))(*[_Shape(r, c) for r, c in mats])
    return int(_lib.vpps_paper_choose_cps(sh, len(mats), n_sm, tb, rpw, int(pack_rows)))


def to_csr(graphs):
    """Graphs as lists of (children, token, label[, chars]) -> CSR int32 arrays of vpps_batch (the last two,
    the BiLSTMwChar spellings, are None when no node has a fourth element)."""
    nodes = [n for g in graphs for n in g]
    nn = len(nodes)
    gp = np.zeros(len(graphs) + 1, np.int32)
    np.cumsum(np.fromiter((len(g) for g in graphs), np.int32, len(graphs)), out=gp[1:])
    cp = np.zeros(nn + 1, np.int32)
    np.cumsum(np.fromiter((len(n[0]) for n in nodes), np.int32, nn), out=cp[1:])
    ch = np.fromiter(itertools.chain.from_iterable(n[0] for n in nodes), np.int32, int(cp[-1]))
    tok = np.fromiter((n[1] for n in nodes), np.int32, nn)
    lab = np.fromiter((n[2] for n in nodes), np.int32, nn)
    chp = chs = None
    if any(len(n) > 3 for n in nodes):
        chp = np.zeros(nn + 1, np.int32)
        np.cumsum(np.fromiter((len(n[3]) if len(n) > 3 else 0 for n in nodes), np.int32, nn), out=chp[1:])
        chs = np.fromiter(itertools.chain.from_iterable(n[3] for n in nodes if len(n) > 3), np.int32, int(chp[-1]))
        chs = chs if chs.size else np.zeros(1, np.int32)
    return gp, cp, ch if ch.size else np.zeros(1, np.int32), tok, lab, chp, chs


class CsrBatch:
    """A batch in the CSR form of vpps_batch (include/vpps.h): graph_ptr, child_ptr, children, token, label."""

    def __init__(self, graph_ptr, child_ptr, children, token, label, char_ptr=None, chars=None):
        as32 = lambda a: np.ascontiguousarray(np.asarray(a, dtype=np.int32))
        self.arrays = (as32(graph_ptr), as32(child_ptr), as32(children), as32(token), as32(label))
        self.chars = (as32(char_ptr), as32(chars)) if char_ptr is not None else (None, None)

    @classmethod
    def from_graphs(cls, graphs):
        return cls(*to_csr(graphs))


def prefetch_scripts(model: "Model", batches, depth: int = 4, workers: int = 3, executor=None):
    """Yield model.build_script(b) for b in batches, in order, built up to `depth` ahead by `workers`
    background threads (the C++ builder runs without the GIL), so host script generation
    overlaps the device passes: one builder takes ~100-200 us per 16-tree batch, about a device step.
    `executor`: an existing concurrent.futures executor to build on (kept running across calls)."""
    import collections
    import contextlib
    from concurrent.futures import ThreadPoolExecutor
    it = iter(batches)
    own = executor is None
    with (ThreadPoolExecutor(max_workers=max(1, workers)) if own else contextlib.nullcontext(executor)) as ex:
        pend = collections.deque()
        for b in it:
            pend.append(ex.submit(model.build_script, b))
            if len(pend) >= depth:
                break
        while pend:
            s = pend.popleft().result()      # re-raises a builder error in the consumer
            for b in it:
                pend.append(ex.submit(model.build_script, b))
                break
            yield s


# ---- profile-guided choice of the device path (kernels are built for several register
#      layouts and the one to use is picked by timing batches) ----
def candidate_options(cell: str, H: int, C: int):
    """The device paths this build offers for an op set (vpps_define_model options), paper order first."""
    out = []
    if cell == "binary":
        if H == 256:
            out += [dict(cluster=16, dataflow=True), dict(cluster=16)]
        elif H == 128:
            out += [dict(cluster=8, dataflow=True)]          # groups of H / 16 CTAs
        out += [dict(groups=g, level=-1) for g in (4, 2, 1)] + [dict(level=1)]
    elif cell == "childsum":
        out += [dict(groups=g) for g in (4, 2, 1)]
    elif cell == "lstm":
        if C <= 32:
            out += [dict(groups=g, level=-1) for g in (1, 2)]
        out += [dict(level=1, chain=0), dict(level=1, chain=-1)]
    elif cell in ("gru", "bilstm"):
        out += [dict(chain=0), dict(chain=-1)]
    else:
        out += [dict()]
    return out


def autotune(cell: str, H: int, E: int, C: int, batches, inputs, candidates=None, mlp: int = 256, device: int = 0,
             warmup: int = 2, reps: int = 3, timer=None):
    """Time one training pass per sample batch on every candidate path and return (best options, {options
    repr: ms per pass}).  Candidates that this build cannot instantiate (VPPS_E_NOFIT / INVALID) are skipped.
    `timer(model, scripts, inputs)` -> ms overrides the CUDA-event timing (tests)."""
    import torch
    results = {}
    best, best_ms = None, float("inf")
    for opts in (candidates if candidates is not None else candidate_options(cell, H, C)):
        try:
            m = Model(cell, H, E, C, device=device, mlp=mlp, **opts)
        except VppsError:
            continue
        if timer is not None:
            ms = timer(m, batches, inputs)
        else:
            params = torch.zeros(m.n_floats, dtype=torch.float32, device=f"cuda:{device}")
            torch.nn.init.uniform_(params, -0.05, 0.05)
            grads = torch.zeros_like(params)
            m.bind(params, grads)
            scripts = [m.build_script(b) for b in batches]
            for s in scripts:
                s.upload()
            for _ in range(warmup):
                for s in scripts:
                    m.fwd_bwd(s, inputs)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record()
            for _ in range(reps):
                for s in scripts:
                    m.fwd_bwd(s, inputs)
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / (reps * len(scripts))
        results[repr(opts)] = ms
        if ms < best_ms:
            best, best_ms = opts, ms
    if best is None:
        raise VppsError(-2, "no candidate device path for this op set")
    return best, results


class Script:
    def __init__(self, model: "Model", handle: ct.c_void_p):
        self._model = model
        self._h = handle

    @property
    def handle(self):
        return self._h

    def words(self) -> np.ndarray:
        p = ct.POINTER(ct.c_uint32)()
        n = ct.c_int64()
        _check(_lib.vpps_script_words(self._h, ct.byref(p), ct.byref(n)))
        return np.ctypeslib.as_array(p, shape=(n.value,)).copy() if n.value else np.zeros(0, np.uint32)

    def blob(self):
        """(device upload blob as uint32 array, offset of the device lowering, offset of the dataflow
        program or -1) — SPEC_SCRIPT.md §D."""
        p = ct.POINTER(ct.c_uint32)()
        n, lo, do = ct.c_int64(), ct.c_int64(), ct.c_int64()
        _check(_lib.vpps_script_blob(self._h, ct.byref(p), ct.byref(n), ct.byref(lo), ct.byref(do)))
        arr = np.ctypeslib.as_array(p, shape=(n.value,)).copy() if n.value else np.zeros(0, np.uint32)
        return arr, lo.value, do.value

    def info(self) -> dict:
        i = _Info()
        _check(_lib.vpps_script_info_get(self._h, ct.byref(i)))
        return {f: getattr(i, f) for f, _ in _Info._fields_}

    def upload(self, stream=None):
        _check(_lib.vpps_upload_script(self._h, _stream_ptr(stream)))

    def __del__(self):
        if getattr(self, "_h", None) and _lib is not None:   # _lib is None during interpreter shutdown
            _lib.vpps_destroy_script(self._h)
            self._h = None


class Model:
    """vpps_define_model + vpps_bind_buffers (`vpps::handle hndl(model)`)."""

    def __init__(self, cell: str, H: int, E: int, C: int, device: int = 0, n_sm: int = 0, groups: int = 1,
                 plan_only: bool = False, cluster: int = 0, dataflow: bool = False, level: int = 0,
                 mlp: int = 256, allocator: str = "torch", chain: int = 0, Ec: int = 64, Vc: int = 64):
        """allocator: "torch" (the library's device buffers come from torch's caching allocator) or
        "cuda" (the library's default, stream-ordered cudaMallocAsync)."""
        self.cell, self.H, self.E, self.C = cell, H, E, C
        self.shapes = param_shapes(cell, H, E, C, mlp, Ec, Vc)
        sh = (_Shape * len(self.shapes))(*[_Shape(s[0], s[1] if len(s) == 2 else 1) for _, s in self.shapes])
        ops = _Opset(CELLS[cell], E, H, C, mlp)
        self._alloc_cbs = _torch_allocator(device) if (allocator == "torch" and not plan_only) else \
            (_ALLOC_FN(), _FREE_FN())
        opt = _Options(n_sm, 1, groups, device, int(plan_only), cluster, int(dataflow), int(level), int(chain),
                       self._alloc_cbs[0], self._alloc_cbs[1], None)
        self.options = dict(groups=groups, cluster=cluster, dataflow=dataflow, level=level, chain=chain)
        h = ct.c_void_p()
        _check(_lib.vpps_define_model(sh, len(self.shapes), ct.byref(ops), ct.byref(opt), ct.byref(h)))
        self._h = h
        n = ct.c_int64()
        offs = (ct.c_int64 * len(self.shapes))()
        _check(_lib.vpps_layout(self._h, ct.byref(n), offs))
        self.n_floats = n.value
        self.offsets = list(offs)
        self._bound = None

    # ---- layout helpers (views into a flat buffer) ----
    def views(self, flat):
        out = {}
        for (name, shape), o in zip(self.shapes, self.offsets):
            size = int(np.prod(shape))
            out[name] = flat[o:o + size].view(*shape) if hasattr(flat, "view") and not isinstance(flat, np.ndarray) \
                else flat[o:o + size].reshape(shape)
        return out

    def bind(self, params, grads):
        """params/grads: contiguous float32 CUDA tensors of n_floats (caller-owned)."""
        assert params.is_cuda and grads.is_cuda and params.dtype == grads.dtype
        assert params.numel() == self.n_floats and grads.numel() == self.n_floats
        _check(_lib.vpps_bind_buffers(self._h, ct.c_void_p(params.data_ptr()), ct.c_void_p(grads.data_ptr())))
        self._bound = (params, grads)

    def partition_table(self) -> np.ndarray:
        p = ct.POINTER(ct.c_int32)()
        n = ct.c_int64()
        _check(_lib.vpps_partition_table(self._h, ct.byref(p), ct.byref(n)))
        return np.ctypeslib.as_array(p, shape=(n.value * 8,)).reshape(n.value, 8).copy()

    def plan_info(self) -> dict:
        a, b, c, d = ct.c_int32(), ct.c_int32(), ct.c_int32(), ct.c_int32()
        _check(_lib.vpps_plan_info(self._h, ct.byref(a), ct.byref(b), ct.byref(c), ct.byref(d)))
        return dict(n_cta=a.value, n_g=b.value, n_act=c.value, umax=d.value)

    def build_script(self, graphs) -> Script:
        """graphs: a list of graphs (lists of (children, token, label)) or a CsrBatch (to_csr output, the
        form a data loader hands over: no per-node Python work)."""
        csr = graphs if isinstance(graphs, CsrBatch) else CsrBatch(*to_csr(graphs))
        gp, cp, ch, tok, lab = csr.arrays
        chp, chs = csr.chars
        b = _Batch(len(gp) - 1, gp.ctypes.data, cp.ctypes.data, ch.ctypes.data, tok.ctypes.data, lab.ctypes.data,
                   chp.ctypes.data if chp is not None else None, chs.ctypes.data if chs is not None else None)
        h = ct.c_void_p()
        _check(_lib.vpps_build_script(self._h, ct.byref(b), ct.byref(h)))
        return Script(self, h)

    def fwd_bwd(self, script: Script, inputs, d_inputs=None, stream=None):
        _check(_lib.vpps_fwd_bwd(self._h, script.handle, ct.c_void_p(inputs.data_ptr()), inputs.shape[0],
                                 ct.c_void_p(d_inputs.data_ptr()) if d_inputs is not None else None,
                                 _stream_ptr(stream)))

    def fwd_bwd_sgd(self, script: Script, inputs, d_inputs=None, lr=0.0, weight_decay=0.0, stream=None):
        _check(_lib.vpps_fwd_bwd_sgd(self._h, script.handle, ct.c_void_p(inputs.data_ptr()), inputs.shape[0],
                                     ct.c_void_p(d_inputs.data_ptr()) if d_inputs is not None else None,
                                     lr, weight_decay, _stream_ptr(stream)))

    def sgd_step(self, lr: float, weight_decay: float = 0.0, stream=None):
        _check(_lib.vpps_sgd_step(self._h, lr, weight_decay, _stream_ptr(stream)))

    def stale_loss(self) -> float:
        v = ct.c_float()
        _check(_lib.vpps_get_stale_loss(self._h, ct.byref(v)))
        return v.value

    def latest_loss(self) -> float:
        v = ct.c_float()
        _check(_lib.vpps_sync_get_latest_loss(self._h, ct.byref(v)))
        return v.value

    def set_timing_events(self, before, after):
        """torch.cuda.Event pair recorded around every later kernel launch (None clears)."""
        _check(_lib.vpps_set_timing_events(self._h, ct.c_void_p(before.cuda_event) if before else None,
                                           ct.c_void_p(after.cuda_event) if after else None))

    def set_kernel_events(self, before, after):
        """torch.cuda.Event pair recorded around the replica-group kernel alone (None clears)."""
        _check(_lib.vpps_set_kernel_events(self._h, ct.c_void_p(before.cuda_event) if before else None,
                                           ct.c_void_p(after.cuda_event) if after else None))

    def set_gemm_trace(self, buf=None):
        """int64 CUDA tensor [items, 5] receiving (group, item, start ns, end ns, smid) per GEMM item."""
        _check(_lib.vpps_set_gemm_trace(self._h, ct.c_void_p(buf.data_ptr()) if buf is not None else None))

    def set_profile_buffer(self, buf=None, stride=0):
        """int64 CUDA tensor [n_cta, stride] receiving the in-kernel globaltimer trace (None clears)."""
        _check(_lib.vpps_set_profile_buffer(self._h, ct.c_void_p(buf.data_ptr()) if buf is not None else None,
                                            stride))

    def pool(self):
        """(device pointer, words) of the activation pool of the last pass."""
        p, n = ct.c_void_p(), ct.c_int64()
        _check(_lib.vpps_pool_ptr(self._h, ct.byref(p), ct.byref(n)))
        return p.value, n.value

    def __del__(self):
        if getattr(self, "_h", None) and _lib is not None:
            _lib.vpps_destroy_model(self._h)
            self._h = None
