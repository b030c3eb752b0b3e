"""Thin Python binding of the Astra B200 C-ABI library (include/astra.h).

Argument marshalling only: every step of the training path runs in the library's CUDA kernels
(lib/libastra.so, built for sm_100a by build.py).  PyTorch is used for device memory, streams
and process groups.  There is NO CPU fallback: if the library is missing or a call fails, an
exception is raised.
"""
from __future__ import annotations

import ctypes
import json
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "lib", "libastra.so")

LSTM, MILSTM, SCRNN, RHN, LSTM_ATTN, SUBLSTM = 0, 1, 2, 3, 4, 5
CELL_TYPES = {"lstm": LSTM, "milstm": MILSTM, "scrn": SCRNN, "rhn": RHN, "attn": LSTM_ATTN, "sublstm": SUBLSTM}
BF16, FP32 = 0, 1
TUNE_OFF, TUNE_ON, TUNE_FROZEN = 0, 1, 2
TUNE_IDLE, TUNE_EXPLORING, TUNE_CONVERGED = 0, 1, 2


class AstraError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{msg} [status {status}]")
        self.status = status


class CellDesc(ctypes.Structure):
    _fields_ = [("cell_type", ctypes.c_int), ("hidden", ctypes.c_int), ("input", ctypes.c_int),
                ("batch", ctypes.c_int), ("seq", ctypes.c_int), ("dtype", ctypes.c_int),
                ("device", ctypes.c_int), ("depth", ctypes.c_int), ("context", ctypes.c_int),
                ("scrn_alpha", ctypes.c_float), ("src_seq", ctypes.c_int), ("attn_dim", ctypes.c_int)]


FAKE_COST = ctypes.CFUNCTYPE(None, ctypes.POINTER(ctypes.c_int), ctypes.c_int, ctypes.POINTER(ctypes.c_double),
                             ctypes.c_int, ctypes.c_void_p)

_lib = None

_P, _I, _SZ, _F = ctypes.c_void_p, ctypes.c_int, ctypes.c_size_t, ctypes.c_float
_SIGS = {
    "astra_cell_create": [ctypes.POINTER(_P), _I, _I, _I, _I, _I],
    "astra_cell_create_ex": [ctypes.POINTER(_P), ctypes.POINTER(CellDesc)],
    "astra_cell_destroy": [_P],
    "astra_param_count": [_P, ctypes.POINTER(_SZ)],
    "astra_param_info": [_P, _I, ctypes.POINTER(ctypes.c_char_p), ctypes.POINTER(_SZ), ctypes.POINTER(_I),
                         ctypes.POINTER(_I)],
    "astra_workspace_size": [_P, ctypes.POINTER(_SZ), ctypes.POINTER(_SZ)],
    "astra_bind": [_P, _P, _P, _P, _P],
    "astra_set_streams": [_P, _P, ctypes.POINTER(_P), _I, _P],
    "astra_step_fwd": [_P, _P, _P, _P, _P, _P, _P],
    "astra_step_bwd": [_P, _P, _P, _P, _P, _P, _P],
    "astra_sgd": [_P, _F],
    "astra_tune_next": [_P, ctypes.POINTER(_I)],
    "astra_tune_mode": [_P, _I, ctypes.c_char_p],
    "astra_tune_report": [_P, ctypes.c_char_p, _SZ, ctypes.POINTER(_SZ)],
    "astra_set_profiling": [_P, _I],
    "astra_comm_init": [_P, _P, _I, _I],
    "astra_lm_comm_init": [_P, _P, _I, _I],
    "astra_comm_unique_id": [_P, _SZ],
    "astra_comm_peer_handle": [_P, _P, _SZ],
    "astra_comm_peer_init": [_P, _P, _I, _I],
    "astra_lm_comm_peer_handle": [_P, _P, _SZ],
    "astra_lm_comm_peer_init": [_P, _P, _I, _I],
    "astra_lm_create": [ctypes.POINTER(_P), _P, _I],
    "astra_lm_destroy": [_P],
    "astra_lm_create_stacked": [ctypes.POINTER(_P), _P, _I, _I],
    "astra_lm_param_count": [_P, ctypes.POINTER(_SZ)],
    "astra_lm_param_info": [_P, _I, ctypes.POINTER(ctypes.c_char_p), ctypes.POINTER(_SZ), ctypes.POINTER(_I),
                            ctypes.POINTER(_I)],
    "astra_lm_workspace_size": [_P, ctypes.POINTER(_SZ)],
    "astra_lm_bind": [_P, _P, _P, _P],
    "astra_lm_set_state": [_P, _P, _P],
    "astra_lm_train_step": [_P, _P, _F, _P],
    "astra_lm_fwd_bwd": [_P, _P, _P],
    "astra_lm_set_graph": [_P, _I],
    "astra_lm_set_buckets": [_P, _P, _I],
    "astra_lm_train_step_len": [_P, _P, _I, _F, _P],
    "astra_lm_fwd_bwd_len": [_P, _P, _I, _P],
    "astra_gemm_bf16": [_I, _I, _I, _P, _I, ctypes.c_long, _P, _I, ctypes.c_long, _P, ctypes.c_long, _I, _I, _I, _P],
    "astra_gemm_bf16_ex": [_I, _I, _I, _P, _I, ctypes.c_long, _P, _I, ctypes.c_long, _P, ctypes.c_long, _I, _I, _I,
                           _I, _I, _P],
    "astra_micro_stream_read": [_P, _SZ, _I, _P, _P],
    "astra_micro_grid_barrier": [_P, _I, _P],
    "astra_micro_launch_chain": [_I, _I, _I, _P],
    "astra_micro_tma_read": [_P, ctypes.c_long, _I, _I, _I, _I, _I, _I, _P],
    "astra_micro_mma_chain": [_I, _I, _I, _I, _I, _P, _P, _P],
    "astra_micro_peer_reduce": [_P, _P, _I, _SZ, _I, ctypes.c_uint, _P],
    "astra_debug_set_trace": [_I, _P],
    "astra_status_string": [_I],
    "astra_last_error": [],
    "astra_kernel_launch_count": [],
    "astra_region_times": [_P, ctypes.POINTER(ctypes.c_double), _I, ctypes.POINTER(_I)],
    "astra_tuner_selftest": [ctypes.c_char_p, FAKE_COST, _P, ctypes.POINTER(_I), _I, ctypes.POINTER(_I),
                             ctypes.POINTER(_I), ctypes.POINTER(_I)],
}


def lib():
    """Load lib/libastra.so (raises if it has not been built — no fallback)."""
    global _lib
    if _lib is None:
        path = os.environ.get("ASTRA_LIB_OVERRIDE") or LIB_PATH   # A/B runs against another in-tree build
        if not os.path.exists(path):
            raise ImportError(f"{path} not built: run `python -m paper_conf_asplos_sivathanucsz19_b200.build`")
        L = ctypes.CDLL(path)
        for name, args in _SIGS.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = ctypes.c_int
        L.astra_status_string.restype = ctypes.c_char_p
        L.astra_last_error.restype = ctypes.c_char_p
        L.astra_kernel_launch_count.restype = ctypes.c_uint64
        _lib = L
    return _lib


def _check(st):
    if st != 0:
        L = lib()
        raise AstraError(st, f"{L.astra_status_string(st).decode()}: {L.astra_last_error().decode()}")


def launch_count():
    return int(lib().astra_kernel_launch_count())


def _ptr(t):
    """Raw pointer of a tensor handed to the C ABI, which takes dense row-major buffers only: a
    strided view (e.g. from numpy fancy indexing) would be read in the wrong order, so it is
    refused instead of silently reinterpreted."""
    if t is None:
        return None
    if not t.is_contiguous():
        raise ValueError(f"astra: tensor of shape {tuple(t.shape)} / strides {t.stride()} is not contiguous "
                         "(the C ABI takes dense row-major buffers; call .contiguous())")
    return ctypes.c_void_p(t.data_ptr())


def _stream():
    import torch
    return ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)


def gemm_bf16(A, B, M, N, K, a_mn=False, b_mn=False, bn=256, cm=1, cn=1, out=None):
    """K1 as a library GEMM: out[M, N] fp32 = A·B (see astra_gemm_bf16)."""
    import torch
    if out is None:
        out = torch.empty(M, N, dtype=torch.float32, device=A.device)
    _check(lib().astra_gemm_bf16(M, N, K, _ptr(A), int(a_mn), A.stride(0), _ptr(B), int(b_mn), B.stride(0),
                                 _ptr(out), out.stride(0), bn, cm, cn, _stream()))
    return out


def gemm_bf16_ex(A, B, M, N, K, a_mn=False, b_mn=False, bn=256, cm=1, cn=1, cta_group=1, ksplit=1, out=None):
    """Extended K1 (see astra_gemm_bf16_ex): CTA pairs and fixed split-K.  Returns out[ksplit, M, N]
    fp32 partials (out[0] is the product when ksplit = 1)."""
    import torch
    if out is None:
        out = torch.zeros(ksplit, M, N, dtype=torch.float32, device=A.device)
    _check(lib().astra_gemm_bf16_ex(M, N, K, _ptr(A), int(a_mn), A.stride(0), _ptr(B), int(b_mn), B.stride(0),
                                    _ptr(out), out.stride(1), bn, cm, cn, cta_group, ksplit, _stream()))
    return out


def _alloc_bytes(n, device):
    import torch
    return torch.empty(max(int(n), 256), dtype=torch.uint8, device=device)


class Cell:
    """One recurrent cell instance (astra_cell) with its parameters, gradients and workspace."""

    def __init__(self, cell, hidden, input, batch, seq, dtype="bf16", device=0, depth=0, context=0,
                 scrn_alpha=0.0, src_seq=0, attn_dim=0, allocate=True, side_streams=2):
        import torch
        L = lib()
        self.cell_type = CELL_TYPES[cell] if isinstance(cell, str) else int(cell)
        self.dtype = dtype
        self.device = torch.device("cuda", device) if allocate else None
        d = CellDesc(self.cell_type, hidden, input, batch, seq, BF16 if dtype == "bf16" else FP32, device, depth,
                     context, scrn_alpha, src_seq, attn_dim)
        h = ctypes.c_void_p()
        _check(L.astra_cell_create_ex(ctypes.byref(h), ctypes.byref(d)))
        self.h = h
        self.H, self.I, self.B, self.T = hidden, input, batch, seq
        n = ctypes.c_size_t()
        _check(L.astra_param_count(h, ctypes.byref(n)))
        self.n_params = n.value
        self.param_info = _param_info(L.astra_param_info, h)
        sv, sc = ctypes.c_size_t(), ctypes.c_size_t()
        _check(L.astra_workspace_size(h, ctypes.byref(sv), ctypes.byref(sc)))
        self.saved_bytes, self.scratch_bytes = sv.value, sc.value
        self._streams = []
        if allocate:
            self.params = torch.zeros(self.n_params, dtype=torch.float32, device=self.device)
            self.grads = torch.zeros(self.n_params, dtype=torch.float32, device=self.device)
            self.saved = _alloc_bytes(self.saved_bytes, self.device)
            self.scratch = _alloc_bytes(self.scratch_bytes, self.device)
            _check(L.astra_bind(h, _ptr(self.params), _ptr(self.grads), _ptr(self.saved), _ptr(self.scratch)))
            self.set_streams(side_streams)

    def set_streams(self, n_side=1):
        import torch
        self._side = [torch.cuda.Stream(device=self.device) for _ in range(n_side)]
        arr = (ctypes.c_void_p * max(1, n_side))(*[s.cuda_stream for s in self._side])
        _check(lib().astra_set_streams(self.h, _stream(), arr, n_side, None))

    def set_profiling(self, on):
        """Region cudaEvent pairs (astra_set_profiling): False / 0 off (only outside exploration),
        True / 1 the always-on level (step region; phase regions while exploring), 2 every phase
        region every step (diagnostics)."""
        _check(lib().astra_set_profiling(self.h, int(on)))

    def view(self, name, t=None):
        """View of parameter `name` inside the flat params (or grads) vector, external layout."""
        t = self.params if t is None else t
        off, r, c = self.param_info[name]
        v = t[off:off + r * c]
        return v.view(r, c) if r > 1 else v

    def load(self, named):
        for k, v in named.items():
            import torch
            self.view(k).copy_(torch.as_tensor(v, dtype=torch.float32).reshape(self.view(k).shape))

    def forward(self, x, h0=None, c0=None, y=None, hT=None, cT=None):
        _check(lib().astra_step_fwd(self.h, _ptr(x), _ptr(h0), _ptr(c0), _ptr(y), _ptr(hT), _ptr(cT)))

    def backward(self, dy, dhT=None, dcT=None, dx=None, dh0=None, dc0=None):
        _check(lib().astra_step_bwd(self.h, _ptr(dy), _ptr(dhT), _ptr(dcT), _ptr(dx), _ptr(dh0), _ptr(dc0)))

    def sgd(self, lr):
        _check(lib().astra_sgd(self.h, lr))

    def tune_mode(self, mode, variant=None):
        _check(lib().astra_tune_mode(self.h, mode, None if variant is None else variant.encode()))

    def tune_next(self):
        s = ctypes.c_int()
        _check(lib().astra_tune_next(self.h, ctypes.byref(s)))
        return s.value

    def tune_report(self):
        n = ctypes.c_size_t()
        _check(lib().astra_tune_report(self.h, None, 0, ctypes.byref(n)))
        buf = ctypes.create_string_buffer(n.value)
        _check(lib().astra_tune_report(self.h, buf, n.value, ctypes.byref(n)))
        return json.loads(buf.value.decode())

    def comm_init(self, uid: bytes, rank, world):
        b = ctypes.create_string_buffer(uid, len(uid))
        _check(lib().astra_comm_init(self.h, b, rank, world))

    def comm_peer_handle(self) -> bytes:
        """This rank's peer-memory window handle (astra_comm_peer_handle, K11p)."""
        return _peer_handle(lib().astra_comm_peer_handle, self.h)

    def comm_peer_init(self, handles: bytes, rank, world):
        """Map every rank's window (astra_comm_peer_init); handles = the rank-ordered concatenation."""
        _peer_init(lib().astra_comm_peer_init, self.h, handles, rank, world)

    def __del__(self):
        try:
            if getattr(self, "h", None) and not getattr(self, "_owned", False):
                lib().astra_cell_destroy(self.h)
        except Exception:
            pass


PEER_HANDLE_BYTES = 256   # ASTRA_PEER_HANDLE_BYTES


def _peer_handle(fn, h):
    b = ctypes.create_string_buffer(PEER_HANDLE_BYTES)
    _check(fn(h, b, PEER_HANDLE_BYTES))
    return b.raw


def _peer_init(fn, h, handles, rank, world):
    assert len(handles) == world * PEER_HANDLE_BYTES, "handles: world x PEER_HANDLE_BYTES bytes in rank order"
    b = ctypes.create_string_buffer(bytes(handles), len(handles))
    _check(fn(h, b, rank, world))


def peer_exchange(obj, group=None):
    """Set up the deterministic peer-memory DP backend (K11p) of `obj` (a Cell or an LM) over a
    torch.distributed process group: all-gather the ranks' window handles in rank order, then map
    them.  Host plumbing only — the gradient sum and SGD run in the library's kernels."""
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    mine = obj.comm_peer_handle()
    allh = [None] * world
    dist.all_gather_object(allh, mine, group=group)
    obj.comm_peer_init(b"".join(allh), rank, world)
    return rank, world


def comm_unique_id() -> bytes:
    b = ctypes.create_string_buffer(128)
    _check(lib().astra_comm_unique_id(b, 128))
    return b.raw


def _param_info(fn, h):
    out = {}
    i = 0
    while True:
        nm, off, r, c = ctypes.c_char_p(), ctypes.c_size_t(), ctypes.c_int(), ctypes.c_int()
        st = fn(h, i, ctypes.byref(nm), ctypes.byref(off), ctypes.byref(r), ctypes.byref(c))
        if st != 0:
            break
        out[nm.value.decode()] = (off.value, r.value, c.value)
        i += 1
    return out


class LM:
    """Embedding → cell → linear head → mean cross-entropy, with SGD (astra_lm)."""

    def __init__(self, cell, vocab: int):
        """cell: one Cell, or a list of Cells stacked bottom first (astra_lm_create_stacked)."""
        import torch
        L = lib()
        self.layers = list(cell) if isinstance(cell, (list, tuple)) else [cell]
        self.cell = self.layers[-1]
        cell = self.cell
        self.V = vocab
        h = ctypes.c_void_p()
        if len(self.layers) == 1:
            _check(L.astra_lm_create(ctypes.byref(h), cell.h, vocab))
        else:
            arr = (ctypes.c_void_p * len(self.layers))(*[c.h.value for c in self.layers])
            _check(L.astra_lm_create_stacked(ctypes.byref(h), ctypes.cast(arr, ctypes.c_void_p), len(self.layers),
                                             vocab))
        self.h = h
        n = ctypes.c_size_t()
        _check(L.astra_lm_param_count(h, ctypes.byref(n)))
        self.n_params = n.value
        self.param_info = _param_info(L.astra_lm_param_info, h)
        w = ctypes.c_size_t()
        _check(L.astra_lm_workspace_size(h, ctypes.byref(w)))
        self.ws_bytes = w.value
        dev = cell.device
        self.params = torch.zeros(self.n_params, dtype=torch.float32, device=dev)
        self.grads = torch.zeros(self.n_params, dtype=torch.float32, device=dev)
        self.ws = _alloc_bytes(self.ws_bytes, dev)
        self.loss = torch.zeros(1, dtype=torch.float32, device=dev)
        _check(L.astra_lm_bind(h, _ptr(self.params), _ptr(self.grads), _ptr(self.ws)))
        # the LM carved every layer's saved / scratch workspace out of its own: the cells' own
        # buffers (GBs at cfg5) are dead from here on
        for c in self.layers:
            c.saved = c.scratch = None

    def view(self, name, t=None):
        t = self.params if t is None else t
        off, r, c = self.param_info[name]
        v = t[off:off + r * c]
        return v.view(r, c) if r > 1 else v

    def load(self, named):
        import torch
        for k, v in named.items():
            self.view(k).copy_(torch.as_tensor(v, dtype=torch.float32).reshape(self.view(k).shape))

    def set_state(self, h=None, c=None):
        _check(lib().astra_lm_set_state(self.h, _ptr(h), _ptr(c)))

    def train_step(self, tokens, lr, loss=None):
        _check(lib().astra_lm_train_step(self.h, _ptr(tokens), lr, _ptr(self.loss if loss is None else loss)))
        return self.loss if loss is None else loss

    def set_buckets(self, sizes):
        """Bucketed profiling of variable-length mini-batches (astra_lm_set_buckets)."""
        arr = (ctypes.c_int * max(1, len(sizes)))(*sizes)
        _check(lib().astra_lm_set_buckets(self.h, ctypes.cast(arr, ctypes.c_void_p), len(sizes)))

    def train_step_len(self, tokens, length, lr, loss=None):
        """One step on tokens [length+1, B] run at the bucket of `length` (astra_lm_train_step_len)."""
        _check(lib().astra_lm_train_step_len(self.h, _ptr(tokens), int(length), lr,
                                             _ptr(self.loss if loss is None else loss)))
        return self.loss if loss is None else loss

    def fwd_bwd_len(self, tokens, length, loss=None):
        _check(lib().astra_lm_fwd_bwd_len(self.h, _ptr(tokens), int(length), _ptr(self.loss if loss is None else loss)))
        return self.loss if loss is None else loss

    def set_graph(self, on: bool):
        """CUDA-graph replay of frozen steps (see astra_lm_set_graph)."""
        _check(lib().astra_lm_set_graph(self.h, int(bool(on))))

    def fwd_bwd(self, tokens, loss=None):
        _check(lib().astra_lm_fwd_bwd(self.h, _ptr(tokens), _ptr(self.loss if loss is None else loss)))
        return self.loss if loss is None else loss

    def comm_init(self, uid: bytes, rank, world):
        """One NCCL communicator for every layer of the LM (astra_lm_comm_init)."""
        b = ctypes.create_string_buffer(uid, len(uid))
        _check(lib().astra_lm_comm_init(self.h, b, rank, world))

    def comm_peer_handle(self) -> bytes:
        """This rank's peer-memory window handle for the LM's params / grads (K11p)."""
        return _peer_handle(lib().astra_lm_comm_peer_handle, self.h)

    def comm_peer_init(self, handles: bytes, rank, world):
        _peer_init(lib().astra_lm_comm_peer_init, self.h, handles, rank, world)

    def __del__(self):
        try:
            if getattr(self, "h", None):
                lib().astra_lm_destroy(self.h)
        except Exception:
            pass


def tuner_selftest(tree: str, cost, max_trials=100000):
    """Run the native wirer on a fake clock: cost(config list) -> list of metric values."""
    res = {}

    @FAKE_COST
    def cb(cfg, n, out, nm, user):
        vals = cost([cfg[i] for i in range(n)])
        for i in range(nm):
            out[i] = vals[i]
    trials = (ctypes.c_int * (max_trials * 64))()
    nt, na = ctypes.c_int(), ctypes.c_int()
    final = (ctypes.c_int * 64)()
    _check(lib().astra_tuner_selftest(tree.encode(), cb, None, trials, max_trials, ctypes.byref(nt), final,
                                      ctypes.byref(na)))
    n, a = nt.value, na.value
    res["trials"] = [[trials[k * a + i] for i in range(a)] for k in range(min(n, max_trials))]
    res["n_trials"] = n
    res["final"] = [final[i] for i in range(a)]
    return res
