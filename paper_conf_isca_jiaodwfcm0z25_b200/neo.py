"""Thin ctypes binding of libneo.so (include/neo.h).  Argument marshalling only: every step
of the key-switching path runs in the library's CUDA kernels.  There is no fallback -- if
libneo.so is missing or a call fails, this module raises.

Tensors are torch.uint64 CUDA tensors (device memory and streams come from PyTorch); the
functions carry the C names of neo.h and take the same arguments, with (pointer, size)
pairs replaced by tensors.
"""
from __future__ import annotations

import ctypes
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libneo.so")

NEO_OP_KEYSWITCH, NEO_OP_HMULT, NEO_OP_HROT, NEO_OP_RESCALE, NEO_OP_HROT_HOISTED = 0, 1, 2, 3, 4
NEO_NTT_FP64, NEO_NTT_TC = 0, 1
NEO_OP_DOUBLE_RESCALE, NEO_OP_MODRAISE, NEO_OP_HMULT_RESCALE, NEO_OP_HROT_SUM = 5, 6, 7, 8
_STATUS = {0: "NEO_OK", 1: "NEO_EINVAL", 2: "NEO_EUNSUPPORTED", 3: "NEO_ENOMEM", 4: "NEO_ECUDA",
           5: "NEO_ENCCL", 6: "NEO_ENOPRIME"}

EXPORTED = ("neo_params_create", "neo_params_destroy", "neo_params_query", "neo_workspace_size",
            "neo_ntt", "neo_intt", "neo_bconv", "neo_tensor", "neo_automorphism", "neo_evk_create",
            "neo_evk_destroy", "neo_keyswitch", "neo_hmult", "neo_hrot", "neo_rescale",
            "neo_keyip", "neo_moddown_combine", "neo_evk_create_hoisted", "neo_hrot_hoisted",
            "neo_last_error", "neo_last_launch_count", "neo_profile_enable", "neo_profile_read",
            "neo_debug_bconv_trace", "neo_double_rescale", "neo_pmult", "neo_hadd", "neo_padd",
            "neo_evk_create_klss", "neo_klss_query", "neo_profile_timeline", "neo_hsub", "neo_modraise",
            "neo_drop_levels", "neo_pmult_acc", "neo_wire_bytes", "neo_wire_pack", "neo_wire_unpack", "neo_hmult_rescale", "neo_ew_limbs", "neo_hrot_sum",
            "neo_ntt_select", "neo_ntt_selected", "neo_comm_unique_id", "neo_comm_create",
            "neo_comm_create_local", "neo_comm_destroy", "neo_comm_limbs", "neo_workspace_size_sharded",
            "neo_keyswitch_sharded", "neo_query_ql_inv")
PROFILE_KINDS = ("ntt_col", "ntt_row", "bconv", "keyip", "combine", "tensor", "automorphism",
                 "rescale_modswitch", "rescale_combine", "elementwise")


class NeoError(RuntimeError):
    def __init__(self, status: int, where: str, msg: str):
        super().__init__(f"{where}: {_STATUS.get(status, status)}: {msg}")
        self.status = status


class ParamsDesc(ctypes.Structure):
    _fields_ = [("log_n", ctypes.c_int32), ("num_q", ctypes.c_int32), ("num_p", ctypes.c_int32),
                ("dnum", ctypes.c_int32), ("word_bits", ctypes.c_int32), ("device", ctypes.c_int32),
                ("q", ctypes.POINTER(ctypes.c_uint64)), ("p", ctypes.POINTER(ctypes.c_uint64)),
                ("alpha_t", ctypes.c_int32),
                ("word_bits_t", ctypes.c_int32)]


_lib = None
_vp, _i32, _u32, _sz = ctypes.c_void_p, ctypes.c_int32, ctypes.c_uint32, ctypes.c_size_t
_i32p = ctypes.POINTER(ctypes.c_int32)
_u64p = ctypes.POINTER(ctypes.c_uint64)


def lib() -> ctypes.CDLL:
    """Load libneo.so (built by paper_conf_isca_jiaodwfcm0z25_b200.build); raise if absent."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is not built (run python -m paper_conf_isca_jiaodwfcm0z25_b200.build)")
        L = ctypes.CDLL(LIB_PATH)
        sig = {
            "neo_params_create": [ctypes.POINTER(ParamsDesc), ctypes.POINTER(_vp)],
            "neo_params_destroy": [_vp],
            "neo_params_query": [_vp, _u64p, _u64p, _u64p],
            "neo_ntt": [_vp, _vp, _i32p, _i32, _i32, _vp, _sz, _vp],
            "neo_intt": [_vp, _vp, _i32p, _i32, _i32, _vp, _sz, _vp],
            "neo_bconv": [_vp, _vp, _i32p, _i32, _vp, _i32p, _i32, _i32, _vp],
            "neo_query_ql_inv": [_vp, _i32, _i32p, _i32, _u64p],
            "neo_tensor": [_vp, _vp, _vp, _i32, _vp, _i32, _vp],
            "neo_automorphism": [_vp, _vp, _i32, _u32, _vp, _i32, _vp],
            "neo_evk_create": [_vp, _vp, ctypes.POINTER(_vp)],
            "neo_evk_destroy": [_vp],
            "neo_keyswitch": [_vp, _vp, _vp, _i32, _vp, _vp, _i32, _vp, _sz, _vp],
            "neo_hmult": [_vp, _vp, _vp, _vp, _i32, _vp, _i32, _vp, _sz, _vp],
            "neo_hrot_sum": [_vp, ctypes.POINTER(_vp), ctypes.POINTER(_u32), _i32, ctypes.POINTER(_vp), _i32, _vp,
                             _i32, _vp, _sz, _vp],
            "neo_ew_limbs": [_vp, _i32, _vp, _vp, _i32p, _i32, _u64p, _i32, _vp, _i32, _vp],
            "neo_hmult_rescale": [_vp, _vp, _vp, _vp, _i32, _vp, _i32, _vp, _sz, _vp],
            "neo_hrot": [_vp, _vp, _u32, _vp, _i32, _vp, _i32, _vp, _sz, _vp],
            "neo_rescale": [_vp, _vp, _i32, _vp, _i32, _vp, _sz, _vp],
            "neo_keyip": [_vp, _vp, _vp, _i32p, _i32, _i32, _vp, _i32, _vp],
            "neo_evk_create_hoisted": [_vp, _vp, _u32, ctypes.POINTER(_vp)],
            "neo_hrot_hoisted": [_vp, ctypes.POINTER(_vp), _i32, _vp, _i32, _vp, _i32, _vp, _sz, _vp],
            "neo_moddown_combine": [_vp, _vp, _vp, _i32p, _i32, _vp, _i32, _vp],
            "neo_double_rescale": [_vp, _vp, _i32, _vp, _i32, _vp, _sz, _vp],
            "neo_pmult": [_vp, _vp, _vp, _i32, _vp, _i32, _vp],
            "neo_hadd": [_vp, _vp, _vp, _i32, _vp, _i32, _vp],
            "neo_padd": [_vp, _vp, _vp, _i32, _vp, _i32, _vp],
            "neo_evk_create_klss": [_vp, _vp, ctypes.POINTER(_vp)],
            "neo_hsub": [_vp, _vp, _vp, _i32, _vp, _i32, _vp],
            "neo_modraise": [_vp, _vp, _i32, _vp, _i32, _vp, _sz, _vp],
            "neo_drop_levels": [_vp, _vp, _i32, _vp, _i32, _i32, _vp],
            "neo_klss_query": [_vp, _i32p, _i32p, _u64p],
            "neo_wire_pack": [_vp, _vp, _vp, _sz, _vp],
            "neo_wire_unpack": [_vp, _vp, _vp, _sz, _vp],
            "neo_pmult_acc": [_vp, ctypes.POINTER(_vp), ctypes.POINTER(_vp), _i32, _i32, _i32, _vp, _i32, _vp],
            "neo_ntt_select": [_vp, _i32],
            "neo_comm_unique_id": [_vp],
            "neo_comm_create": [_vp, _vp, _i32, _i32, ctypes.POINTER(_vp)],
            "neo_comm_create_local": [_vp, _i32, ctypes.POINTER(_vp)],
            "neo_comm_destroy": [_vp],
            "neo_keyswitch_sharded": [_vp, _vp, _vp, _vp, _i32, _vp, _vp, _i32, _vp, _sz, _vp],
            "neo_ntt_selected": [_vp],
        }
        for name, args in sig.items():
            if not hasattr(L, name):        # an older build (A/B runs); tests/test_abi.py requires every symbol
                continue
            f = getattr(L, name)
            f.argtypes = args
            f.restype = ctypes.c_int
        L.neo_wire_bytes.argtypes = [_sz]
        L.neo_wire_bytes.restype = _sz
        if hasattr(L, "neo_comm_limbs"):
            L.neo_comm_limbs.argtypes = [_vp, _i32, _i32p, _i32p, _i32p]
            L.neo_comm_limbs.restype = _i32
            L.neo_workspace_size_sharded.argtypes = [_vp, _i32, _i32]
            L.neo_workspace_size_sharded.restype = _sz
        L.neo_workspace_size.argtypes = [_vp, _i32, _i32, _i32]
        L.neo_workspace_size.restype = _sz
        L.neo_last_error.restype = ctypes.c_char_p
        L.neo_last_error.argtypes = []
        L.neo_last_launch_count.restype = _i32
        L.neo_last_launch_count.argtypes = []
        L.neo_profile_enable.argtypes = [_i32]
        L.neo_profile_enable.restype = ctypes.c_int
        L.neo_profile_read.argtypes = [_i32, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_int32)]
        L.neo_profile_read.restype = ctypes.c_int
        L.neo_debug_bconv_trace.argtypes = [ctypes.POINTER(ctypes.c_ulonglong)]
        L.neo_debug_bconv_trace.restype = _i32
        _lib = L
    return _lib


def _check(status: int, where: str):
    if status != 0:
        raise NeoError(status, where, lib().neo_last_error().decode())


def _ptr(t: torch.Tensor | None):
    if t is None:
        return None
    if t.dtype != torch.uint64 or not t.is_cuda or not t.is_contiguous():
        raise TypeError("expected a contiguous torch.uint64 CUDA tensor")
    return ctypes.c_void_p(t.data_ptr())


def _stream(stream) -> ctypes.c_void_p:
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _ids(ids) -> ctypes.Array:
    ids = [int(i) for i in ids]
    return (ctypes.c_int32 * len(ids))(*ids)


def last_launch_count() -> int:
    return int(lib().neo_last_launch_count())


def neo_profile_enable(on: bool):
    _check(lib().neo_profile_enable(1 if on else 0), "neo_profile_enable")


def neo_profile_read() -> dict:
    """{kind: (total_ms, launches)} for every kernel kind recorded since neo_profile_enable."""
    out = {}
    for k, name in enumerate(PROFILE_KINDS):
        ms, n = ctypes.c_double(), ctypes.c_int32()
        _check(lib().neo_profile_read(k, ctypes.byref(ms), ctypes.byref(n)), "neo_profile_read")
        out[name] = (ms.value, n.value)
    return out


def neo_profile_timeline(max_n: int = 4096):
    """[(kind name, start_ms, end_ms)] of the launches recorded since neo_profile_enable."""
    L = lib()
    k = (ctypes.c_int32 * max_n)()
    a, b = (ctypes.c_float * max_n)(), (ctypes.c_float * max_n)()
    L.neo_profile_timeline.restype = _i32
    L.neo_profile_timeline.argtypes = [_i32, _i32p, ctypes.POINTER(ctypes.c_float), ctypes.POINTER(ctypes.c_float)]
    n = L.neo_profile_timeline(max_n, k, a, b)
    return [(PROFILE_KINDS[k[i]], a[i], b[i]) for i in range(n)]


def neo_debug_bconv_trace():
    """The BConv pipeline trace (NEO_BCONV_DBG=1) as a [2][64][8] list (ModUp, ModDown), or None."""
    buf = (ctypes.c_ulonglong * 1024)()
    if not lib().neo_debug_bconv_trace(buf):
        return None
    v = list(buf)
    return [[v[w * 512 + r * 8: w * 512 + r * 8 + 8] for r in range(64)] for w in range(2)]


class Context:
    """neo_params_create / neo_params_destroy; q, p, psi from neo_params_query."""

    def __init__(self, log_n: int, num_q: int, num_p: int, dnum: int, word_bits: int = 36, device: int = 0,
                 alpha_t: int = 0, word_bits_t: int = 0):
        self.log_n, self.num_q, self.num_p, self.dnum = log_n, num_q, num_p, dnum
        self.N = 1 << log_n
        self.alpha = -(-num_q // dnum)
        d = ParamsDesc(log_n, num_q, num_p, dnum, word_bits, device, None, None, alpha_t, word_bits_t)
        h = ctypes.c_void_p()
        _check(lib().neo_params_create(ctypes.byref(d), ctypes.byref(h)), "neo_params_create")
        self.handle = h
        q = (ctypes.c_uint64 * num_q)()
        p = (ctypes.c_uint64 * num_p)()
        psi = (ctypes.c_uint64 * (num_q + num_p))()
        _check(lib().neo_params_query(h, q, p, psi), "neo_params_query")
        self.q, self.p, self.psi = list(q), list(p), list(psi)
        self.moduli = self.q + self.p
        at, ap = ctypes.c_int32(), ctypes.c_int32()
        if not hasattr(lib(), "neo_klss_query"):     # an older build in an A/B run
            self.alpha_t, self.alpha_p, self.t = 0, 0, []
            return
        _check(lib().neo_klss_query(h, ctypes.byref(at), ctypes.byref(ap), None), "neo_klss_query")
        self.alpha_t, self.alpha_p = at.value, ap.value
        t = (ctypes.c_uint64 * max(1, self.alpha_p))()
        _check(lib().neo_klss_query(h, None, None, t), "neo_klss_query")
        self.t = list(t)[: self.alpha_p]

    def close(self):
        if self.handle:
            lib().neo_params_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def ntt_select(self, impl: int):
        """neo_ntt_select: NEO_NTT_TC (tcgen05 DFT stages) or NEO_NTT_FP64 (CUDA-core butterflies)."""
        _check(lib().neo_ntt_select(self.handle, impl), "neo_ntt_select")

    @property
    def ntt_impl(self) -> int:
        return int(lib().neo_ntt_selected(self.handle))

    def workspace_size(self, op: int, level: int, batch: int) -> int:
        return int(lib().neo_workspace_size(self.handle, op, level, batch))

    def workspace(self, op: int, level: int, batch: int, device="cuda") -> torch.Tensor:
        n = self.workspace_size(op, level, batch)
        if n == 0:
            raise NeoError(1, "neo_workspace_size", "invalid op/level/batch")
        return torch.empty(n // 8, dtype=torch.uint64, device=device)


class EvalKey:
    """neo_evk_create / neo_evk_destroy (device copy of [dnum][2][num_q+num_p][N]);
    with hoisted_galois=g, neo_evk_create_hoisted (key for neo_hrot_hoisted)."""

    def __init__(self, ctx: Context, evk: torch.Tensor, hoisted_galois: int | None = None, klss: bool = False):
        self.ctx = ctx
        h = ctypes.c_void_p()
        if klss:          # neo_evk_create_klss: evk is [2][beta~][dnum][alpha'][N] over the T primes
            _check(lib().neo_evk_create_klss(ctx.handle, _ptr(evk), ctypes.byref(h)), "neo_evk_create_klss")
        elif hoisted_galois is None:
            _check(lib().neo_evk_create(ctx.handle, _ptr(evk), ctypes.byref(h)), "neo_evk_create")
        else:
            _check(lib().neo_evk_create_hoisted(ctx.handle, _ptr(evk), hoisted_galois, ctypes.byref(h)),
                   "neo_evk_create_hoisted")
        self.galois = hoisted_galois
        self.handle = h

    def close(self):
        if self.handle:
            lib().neo_evk_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def neo_ntt(ctx: Context, poly: torch.Tensor, limb_ids, batch: int, ws: torch.Tensor, stream=None):
    _check(lib().neo_ntt(ctx.handle, _ptr(poly), _ids(limb_ids), len(limb_ids), batch, _ptr(ws),
                         ws.numel() * 8, _stream(stream)), "neo_ntt")


def neo_intt(ctx: Context, poly: torch.Tensor, limb_ids, batch: int, ws: torch.Tensor, stream=None):
    _check(lib().neo_intt(ctx.handle, _ptr(poly), _ids(limb_ids), len(limb_ids), batch, _ptr(ws),
                          ws.numel() * 8, _stream(stream)), "neo_intt")


def neo_bconv(ctx: Context, inp: torch.Tensor, in_ids, out: torch.Tensor, out_ids, batch: int, stream=None):
    _check(lib().neo_bconv(ctx.handle, _ptr(inp), _ids(in_ids), len(in_ids), _ptr(out), _ids(out_ids),
                           len(out_ids), batch, _stream(stream)), "neo_bconv")


def neo_query_ql_inv(ctx: Context, level: int, limb_ids) -> list:
    """q_level^-1 mod q_i for the limb ids i < level (the context's Rescale constants)."""
    out = (ctypes.c_uint64 * max(1, len(limb_ids)))()
    _check(lib().neo_query_ql_inv(ctx.handle, level, _ids(limb_ids), len(limb_ids), out), "neo_query_ql_inv")
    return list(out)[: len(limb_ids)]


def neo_tensor(ctx: Context, ct_a, ct_b, level: int, d, batch: int, stream=None):
    _check(lib().neo_tensor(ctx.handle, _ptr(ct_a), _ptr(ct_b), level, _ptr(d), batch, _stream(stream)),
           "neo_tensor")


def neo_automorphism(ctx: Context, inp, n_limbs: int, galois_elt: int, out, batch: int, stream=None):
    _check(lib().neo_automorphism(ctx.handle, _ptr(inp), n_limbs, galois_elt, _ptr(out), batch,
                                  _stream(stream)), "neo_automorphism")


def neo_keyswitch(ctx: Context, evk: EvalKey, d, level: int, out0, out1, batch: int, ws, stream=None):
    _check(lib().neo_keyswitch(ctx.handle, evk.handle, _ptr(d), level, _ptr(out0), _ptr(out1), batch,
                               _ptr(ws), ws.numel() * 8, _stream(stream)), "neo_keyswitch")


def neo_hmult(ctx: Context, relin: EvalKey, ct_a, ct_b, level: int, ct_out, batch: int, ws, stream=None):
    _check(lib().neo_hmult(ctx.handle, relin.handle, _ptr(ct_a), _ptr(ct_b), level, _ptr(ct_out), batch,
                           _ptr(ws), ws.numel() * 8, _stream(stream)), "neo_hmult")


def neo_hmult_rescale(ctx: Context, relin: EvalKey, ct_a, ct_b, level: int, ct_out, batch: int, ws, stream=None):
    """Rescale(HMULT(ct_a, ct_b)) in one call: ct_out [batch][2][level][N]."""
    _check(lib().neo_hmult_rescale(ctx.handle, relin.handle, _ptr(ct_a), _ptr(ct_b), level, _ptr(ct_out), batch,
                                   _ptr(ws), ws.numel() * 8, _stream(stream)), "neo_hmult_rescale")


def neo_hrot(ctx: Context, rotkey: EvalKey, galois_elt: int, ct_in, level: int, ct_out, batch: int, ws,
             stream=None):
    _check(lib().neo_hrot(ctx.handle, rotkey.handle, galois_elt, _ptr(ct_in), level, _ptr(ct_out), batch,
                          _ptr(ws), ws.numel() * 8, _stream(stream)), "neo_hrot")


def neo_rescale(ctx: Context, ct_in, level: int, ct_out, batch: int, ws, stream=None):
    _check(lib().neo_rescale(ctx.handle, _ptr(ct_in), level, _ptr(ct_out), batch, _ptr(ws), ws.numel() * 8,
                             _stream(stream)), "neo_rescale")


def neo_double_rescale(ctx: Context, ct_in, level: int, ct_out, batch: int, ws, stream=None):
    _check(lib().neo_double_rescale(ctx.handle, _ptr(ct_in), level, _ptr(ct_out), batch, _ptr(ws),
                                    ws.numel() * 8, _stream(stream)), "neo_double_rescale")


def neo_pmult(ctx: Context, ct_in, pt, level: int, ct_out, batch: int, stream=None):
    _check(lib().neo_pmult(ctx.handle, _ptr(ct_in), _ptr(pt), level, _ptr(ct_out), batch, _stream(stream)),
           "neo_pmult")


def neo_hadd(ctx: Context, ct_a, ct_b, level: int, ct_out, batch: int, stream=None):
    _check(lib().neo_hadd(ctx.handle, _ptr(ct_a), _ptr(ct_b), level, _ptr(ct_out), batch, _stream(stream)),
           "neo_hadd")


def neo_padd(ctx: Context, ct_in, pt, level: int, ct_out, batch: int, stream=None):
    _check(lib().neo_padd(ctx.handle, _ptr(ct_in), _ptr(pt), level, _ptr(ct_out), batch, _stream(stream)),
           "neo_padd")


def neo_hsub(ctx: Context, ct_a, ct_b, level: int, ct_out, batch: int, stream=None):
    _check(lib().neo_hsub(ctx.handle, _ptr(ct_a), _ptr(ct_b), level, _ptr(ct_out), batch, _stream(stream)),
           "neo_hsub")


def neo_modraise(ctx: Context, ct_in, level: int, ct_out, batch: int, ws, stream=None):
    _check(lib().neo_modraise(ctx.handle, _ptr(ct_in), level, _ptr(ct_out), batch, _ptr(ws), ws.numel() * 8,
                              _stream(stream)), "neo_modraise")


def neo_drop_levels(ctx: Context, ct_in, level_in: int, ct_out, level_out: int, batch: int, stream=None):
    _check(lib().neo_drop_levels(ctx.handle, _ptr(ct_in), level_in, _ptr(ct_out), level_out, batch,
                                 _stream(stream)), "neo_drop_levels")


def neo_keyip(ctx: Context, evk: EvalKey, dhat, limb_ids, beta: int, acc, batch: int, stream=None):
    _check(lib().neo_keyip(ctx.handle, evk.handle, _ptr(dhat), _ids(limb_ids), len(limb_ids), beta, _ptr(acc),
                           batch, _stream(stream)), "neo_keyip")


def neo_moddown_combine(ctx: Context, acc, conv, q_ids, out, batch: int, stream=None):
    _check(lib().neo_moddown_combine(ctx.handle, _ptr(acc), _ptr(conv), _ids(q_ids), len(q_ids), _ptr(out), batch,
                                     _stream(stream)), "neo_moddown_combine")


NEO_EWL_HADD, NEO_EWL_HSUB, NEO_EWL_PMULT, NEO_EWL_PADD, NEO_EWL_TENSOR, NEO_EWL_SUBMUL, NEO_EWL_LIFT = range(7)


def neo_ew_limbs(ctx: Context, op: int, a, b, limb_ids, out, batch: int, scal=None, src_limb: int = 0,
                 stream=None):
    """Element-wise op on the rows limb_ids of a rank's polynomials (include/neo.h)."""
    sc = (ctypes.c_uint64 * len(limb_ids))(*scal) if scal is not None else None
    _check(lib().neo_ew_limbs(ctx.handle, op, _ptr(a), _ptr(b), _ids(limb_ids), len(limb_ids), sc, src_limb,
                              _ptr(out), batch, _stream(stream)), "neo_ew_limbs")


def neo_wire_bytes(n: int) -> int:
    return int(lib().neo_wire_bytes(n))


def _u8ptr(t: torch.Tensor):
    if t.dtype != torch.uint8 or not t.is_cuda or not t.is_contiguous():
        raise TypeError("expected a contiguous torch.uint8 CUDA tensor")
    return ctypes.c_void_p(t.data_ptr())


def neo_wire_pack(ctx: Context, x: torch.Tensor, wire: torch.Tensor, stream=None):
    """u64 residues x (any shape, numel n) -> uint8 wire [neo_wire_bytes(n)] (36-bit format)."""
    _check(lib().neo_wire_pack(ctx.handle, _ptr(x), _u8ptr(wire), x.numel(), _stream(stream)), "neo_wire_pack")


def neo_wire_unpack(ctx: Context, wire: torch.Tensor, x: torch.Tensor, stream=None):
    _check(lib().neo_wire_unpack(ctx.handle, _u8ptr(wire), _ptr(x), x.numel(), _stream(stream)), "neo_wire_unpack")


def neo_pmult_acc(ctx: Context, cts, pts, level: int, ct_out, batch: int, pt_shared: bool = False, stream=None):
    """sum_k PMULT(cts[k], pts[k]) in one launch; pts[k] is [batch][l+1][N] or, with pt_shared,
    one [l+1][N] plaintext for every batch entry."""
    if len(cts) != len(pts):
        raise NeoError(1, "neo_pmult_acc", "cts and pts differ in length")
    ca = (ctypes.c_void_p * len(cts))(*[_ptr(t).value for t in cts])
    pa = (ctypes.c_void_p * len(pts))(*[_ptr(t).value for t in pts])
    _check(lib().neo_pmult_acc(ctx.handle, ca, pa, len(cts), int(pt_shared), level, _ptr(ct_out), batch,
                               _stream(stream)), "neo_pmult_acc")


def neo_hrot_sum(ctx: Context, keys, galois, cts, level: int, ct_out, batch: int, ws, stream=None):
    """sum_k HROTATE(cts[k], galois[k]) with one ModDown (include/neo.h)."""
    n = len(keys)
    if not (len(galois) == len(cts) == n):
        raise NeoError(1, "neo_hrot_sum", "keys, galois and cts differ in length")
    ka = (ctypes.c_void_p * n)(*[k.handle.value for k in keys])
    ga = (ctypes.c_uint32 * n)(*[int(g) for g in galois])
    ca = (ctypes.c_void_p * n)(*[_ptr(t).value for t in cts])
    _check(lib().neo_hrot_sum(ctx.handle, ka, ga, n, ca, level, _ptr(ct_out), batch, _ptr(ws), ws.numel() * 8,
                              _stream(stream)), "neo_hrot_sum")


def neo_hrot_hoisted(ctx: Context, keys, ct_in, level: int, ct_out, batch: int, ws, stream=None):
    arr = (ctypes.c_void_p * len(keys))(*[k.handle.value for k in keys])
    _check(lib().neo_hrot_hoisted(ctx.handle, arr, len(keys), _ptr(ct_in), level, _ptr(ct_out), batch, _ptr(ws),
                                  ws.numel() * 8, _stream(stream)), "neo_hrot_hoisted")


class Comm:
    """A limb-sharded key-switching communicator (neo_comm_create / neo_comm_create_local)."""

    def __init__(self, ctx: Context, handle):
        self.ctx, self.handle = ctx, handle

    @staticmethod
    def unique_id() -> bytes:
        """neo_comm_unique_id: the 128-byte NCCL unique id rank 0 distributes."""
        buf = (ctypes.c_uint8 * 128)()
        _check(lib().neo_comm_unique_id(buf), "neo_comm_unique_id")
        return bytes(buf)

    @classmethod
    def create(cls, ctx: Context, uid: bytes, nranks: int, rank: int) -> "Comm":
        buf = (ctypes.c_uint8 * 128).from_buffer_copy(uid)
        h = ctypes.c_void_p()
        _check(lib().neo_comm_create(ctx.handle, buf, nranks, rank, ctypes.byref(h)), "neo_comm_create")
        return cls(ctx, h)

    @classmethod
    def create_local(cls, ctx: Context, nranks: int) -> list:
        arr = (ctypes.c_void_p * nranks)()
        _check(lib().neo_comm_create_local(ctx.handle, nranks, arr), "neo_comm_create_local")
        return [cls(ctx, ctypes.c_void_p(arr[r])) for r in range(nranks)]

    def limbs(self, level: int):
        """(Q limb ids, P limb ids) this rank owns at `level` (neo_comm_limbs)."""
        q = (ctypes.c_int32 * 64)()
        p = (ctypes.c_int32 * 64)()
        n_p = ctypes.c_int32()
        nq = lib().neo_comm_limbs(self.handle, level, q, p, ctypes.byref(n_p))
        if nq < 0:
            raise NeoError(1, "neo_comm_limbs", "invalid level")
        return list(q)[:nq], list(p)[: n_p.value]

    def workspace(self, level: int, batch: int, device="cuda") -> torch.Tensor:
        n = int(lib().neo_workspace_size_sharded(self.handle, level, batch))
        if n == 0:
            raise NeoError(1, "neo_workspace_size_sharded", "invalid level/batch")
        return torch.empty(n // 8, dtype=torch.uint64, device=device)

    def close(self):
        if self.handle:
            lib().neo_comm_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def neo_keyswitch_sharded(ctx: Context, comm: Comm, evk: EvalKey, d_local, level: int, out0, out1, batch: int, ws,
                          stream=None):
    """One key-switch of this rank's Q limbs (d_local [batch][nq][N]); out0/out1 [batch][nq][N].
    A rank without Q limbs passes None for d_local / out0 / out1."""
    nb = ws.numel() * 8
    _check(lib().neo_keyswitch_sharded(ctx.handle, comm.handle, evk.handle, _ptr(d_local), level, _ptr(out0),
                                       _ptr(out1), batch, _ptr(ws), nb, _stream(stream)), "neo_keyswitch_sharded")
