"""B200-native FEVES inter-prediction hot path: FSBM ME -> INT -> SME.

Thin ctypes binding over ``libfeves_me.so`` (C-ABI in include/feves_me.h).
Argument marshalling only: every arithmetic step runs in the sm_100a kernels
of ``csrc/``.  PyTorch provides device memory and streams.  There is no CPU
fallback: if the library or a CUDA device is missing, every call raises.

Paper: Ilic, Momcilovic, Roma, Sousa, "FEVES: Framework for Efficient Parallel
Video Encoding on Heterogeneous Systems", ICPP 2014 (/root/reference/PAPER.md,
P:6 defines ME/INT/SME; P:51 the MB-row distributions used by ``shard``).
"""
from __future__ import annotations

import ctypes
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("FEVES_LIB") or os.path.join(_HERE, "libfeves_me.so")   # FEVES_LIB: experiment override
N_PART = 41
N_PHASE = 16

ME_OK, ME_EINVAL, ME_ENOMEM, ME_ECUDA, ME_ESTATE = 0, -1, -2, -3, -4

_lib = None


class FevesError(RuntimeError):
    pass


def lib():
    """Load libfeves_me.so (built in-tree by __graft_entry__.build())."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise FevesError(f"{LIB_PATH} missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
        L = ctypes.CDLL(LIB_PATH)
        P, i = ctypes.c_void_p, ctypes.c_int
        L.me_create.restype = P
        L.me_create.argtypes = [i, i, i, i]
        L.me_create_pmv.restype = P
        L.me_create_pmv.argtypes = [i, i, i, i, i]
        L.me_set_pmv.argtypes = [P, P]
        L.me_destroy.argtypes = [P]
        L.me_last_error.restype = i
        L.me_strerror.restype = ctypes.c_char_p
        L.me_strerror.argtypes = [i]
        L.me_set_stream.argtypes = [P, P]
        L.me_set_rows.argtypes = [P, i, i]
        L.me_get_layout.argtypes = [P, P, P, P, P, P]
        L.me_estimate.argtypes = [P, P, P, P, P]
        L.int_interpolate.argtypes = [P, P, P]
        L.sme_refine.argtypes = [P, P, P, P, P, P, P]
        L.me_encode_frame.argtypes = [P, P, P, P, i, P, P, P, P]
        L.me_last_launch_count.argtypes = [P]
        L.me_stream_reset.argtypes = [P]
        L.me_stream_push.argtypes = [P, P, i, P, P, i, P]
        L.me_stream_outputs.argtypes = [P, P, P]
        L.me_stream_join.argtypes = [P]
        u32 = ctypes.c_uint32
        L.me_stream_push_flags.argtypes = [P, P, i, P, P, i, P, P, u32, P, u32]
        L.me_stream_wait_value.argtypes = [P, P, u32]
        L.me_stream_write_value.argtypes = [P, P, u32]
        L.me_sync.argtypes = [P]
        L.me_set_timing.argtypes = [P, i]
        L.me_get_timings.argtypes = [P, P, P, P]
        L.me_set_fused.argtypes = [P, i]
        L.me_set_option.argtypes = [P, i, i]
        L.me_mode_decision.argtypes = [P, P, P, i, P]
        L.me_ipc_export.argtypes = [P, P, P, ctypes.POINTER(ctypes.c_size_t)]
        L.me_ipc_open.argtypes = [P, P, ctypes.c_size_t, ctypes.c_size_t, ctypes.POINTER(ctypes.c_void_p)]
        L.me_ipc_close.argtypes = [P, P]
        for fn in ("me_set_stream", "me_set_rows", "me_get_layout", "me_estimate", "int_interpolate",
                   "sme_refine", "me_encode_frame", "me_last_launch_count", "me_stream_reset",
                   "me_stream_push", "me_stream_outputs", "me_stream_join", "me_sync", "me_stream_push_flags",
                   "me_stream_wait_value", "me_stream_write_value", "me_set_timing", "me_get_timings", "me_set_fused", "me_set_option", "me_mode_decision",
                   "me_ipc_export", "me_ipc_open", "me_ipc_close"):
            getattr(L, fn).restype = i
        _lib = L
    return _lib


def _check(rc):
    if rc != ME_OK:
        raise FevesError(f"libfeves_me: {lib().me_strerror(rc).decode()} ({rc})")


def _dev_u8(t, name):
    if not (isinstance(t, torch.Tensor) and t.is_cuda and t.dtype == torch.uint8 and t.is_contiguous()):
        raise FevesError(f"{name}: expected a contiguous uint8 CUDA tensor")
    return t


def _check_out(mv_shape, mvs, sads, name, device=None, host_ok=False):
    """out= buffers: the C-ABI cannot check sizes, so a wrong-size or wrong-kind buffer
    would become an out-of-bounds device (or, via the async D2H, host) write."""
    n = 1
    for d in mv_shape:
        n *= d
    for t, dt, k in ((mvs, (torch.int16,), 2), (sads, (torch.uint16, torch.int16), 1)):
        if t is None:
            continue
        if not isinstance(t, torch.Tensor) or t.dtype not in dt or not t.is_contiguous() or t.numel() != n * k:
            raise FevesError(f"{name}: expected contiguous {dt[0]} tensors with {n * k} elements "
                             f"(shape {tuple(mv_shape) + ((2,) if k == 2 else ())})")
        if t.is_cuda:
            if device is not None and t.device != device:
                raise FevesError(f"{name}: tensor on {t.device}, context on {device}")
        elif not host_ok:
            raise FevesError(f"{name}: expected CUDA tensors")
        elif not t.is_pinned():
            raise FevesError(f"{name}: host outputs must be pinned (they are written by an async copy)")
    if sads is not None and mvs.is_cuda != sads.is_cuda:
        raise FevesError(f"{name}: both outputs on the device or both on the host")


def _ptrs(ts):
    return (ctypes.c_void_p * len(ts))(*[t.data_ptr() for t in ts])


class MotionEstimator:
    """One libfeves_me context: W x H frames, SA side ``sa_range``, ``n_rf`` RFs.

    MV/SAD tensors have shape [rows, mb_cols, n_rf, 41, 2] int16 and
    [rows, mb_cols, n_rf, 41] uint16 (rows = the current MB-row stripe).
    """

    def __init__(self, width: int, height: int, sa_range: int, n_rf: int, device=None, max_pmv: int = 0):
        if not torch.cuda.is_available():
            raise FevesError("no CUDA device: the FEVES path has no CPU fallback")
        self.device = torch.device("cuda", torch.cuda.current_device() if device is None else
                                   torch.device(device).index or 0)
        with torch.cuda.device(self.device):
            L = lib()
            self._ctx = L.me_create_pmv(width, height, sa_range, n_rf, max_pmv)
            if not self._ctx:
                raise FevesError(f"me_create_pmv({width},{height},{sa_range},{n_rf},{max_pmv}): "
                                 f"{L.me_strerror(L.me_last_error()).decode()}")
        self.width, self.height, self.sa_range, self.n_rf = width, height, sa_range, n_rf
        self.max_pmv = max_pmv
        self._pmv = None
        vals = [ctypes.c_int() for _ in range(5)]
        _check(lib().me_get_layout(self._ctx, *[ctypes.byref(v) for v in vals]))
        self.mb_cols, self.mb_rows, self.sf_pad, self.sf_pitch, self.sf_rows = [v.value for v in vals]
        self.row0, self.row1 = 0, self.mb_rows

    def close(self):
        if getattr(self, "_ctx", None):
            lib().me_destroy(self._ctx)
            self._ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ------------------------------------------------------------ config --
    def set_rows(self, r0: int, r1: int):
        _check(lib().me_set_rows(self._ctx, r0, r1))
        self.row0, self.row1 = r0, r1

    def _bind_stream(self):
        _check(lib().me_set_stream(self._ctx, ctypes.c_void_p(torch.cuda.current_stream(self.device).cuda_stream)))

    @property
    def launches(self) -> int:
        return lib().me_last_launch_count(self._ctx)

    def mv_shape(self):
        return (self.row1 - self.row0, self.mb_cols, self.n_rf, N_PART)

    def sf_shape(self):
        return (N_PHASE, self.sf_rows, self.sf_pitch)

    def new_mvs(self):
        return (torch.empty(self.mv_shape() + (2,), dtype=torch.int16, device=self.device),
                torch.empty(self.mv_shape(), dtype=torch.uint16, device=self.device))

    def new_sf(self):
        return torch.empty(self.sf_shape(), dtype=torch.uint8, device=self.device)

    # ------------------------------------------------------------- calls --
    def estimate(self, cf, rfs, out=None):
        """Integer FSBM ME (me_estimate).  Returns (mvs, sads)."""
        _dev_u8(cf, "cf")
        assert len(rfs) == self.n_rf
        for r in rfs:
            _dev_u8(r, "rf")
        mvs, sads = out if out is not None else self.new_mvs()
        _check_out(self.mv_shape(), mvs, sads, "estimate(out=)", self.device)
        self._bind_stream()
        _check(lib().me_estimate(self._ctx, cf.data_ptr(), _ptrs(rfs), mvs.data_ptr(), sads.data_ptr()))
        return mvs, sads

    def interpolate(self, rf, out=None):
        """INT (int_interpolate): 16 phase planes [16, sf_rows, sf_pitch] u8."""
        _dev_u8(rf, "rf")
        sf = self.new_sf() if out is None else out
        _dev_u8(sf, "interpolate(out=)")
        if sf.numel() != N_PHASE * self.sf_rows * self.sf_pitch:
            raise FevesError(f"interpolate(out=): need {self.sf_shape()} bytes")
        self._bind_stream()
        _check(lib().int_interpolate(self._ctx, rf.data_ptr(), sf.data_ptr()))
        return sf

    def refine(self, cf, sfs, mvs, sads=None, out=None):
        """SME (sme_refine).  Returns (qmvs quarter-pel, sads)."""
        _dev_u8(cf, "cf")
        assert len(sfs) == self.n_rf
        qmvs, qsads = out if out is not None else self.new_mvs()
        _check_out(self.mv_shape(), qmvs, qsads, "refine(out=)", self.device)
        _check_out(self.mv_shape(), mvs, sads, "refine(mvs, sads)", self.device)
        self._bind_stream()
        _check(lib().sme_refine(self._ctx, cf.data_ptr(), _ptrs(sfs), mvs.data_ptr(),
                                None if sads is None else sads.data_ptr(), qmvs.data_ptr(), qsads.data_ptr()))
        return qmvs, qsads

    def encode_frame(self, cf, rfs, sfs, n_int, out_me=None, out_sme=None):
        """INT (first n_int RFs) -> ME -> SME in one C call (me_encode_frame)."""
        qmvs, qsads = out_sme if out_sme is not None else self.new_mvs()
        mvs, sads = out_me if out_me is not None else (None, None)
        _check_out(self.mv_shape(), qmvs, qsads, "encode_frame(out_sme=)", self.device)
        if out_me is not None:
            _check_out(self.mv_shape(), mvs, sads, "encode_frame(out_me=)", self.device)
        self._bind_stream()
        _check(lib().me_encode_frame(self._ctx, cf.data_ptr(), _ptrs(rfs), _ptrs(sfs), n_int,
                                     None if mvs is None else mvs.data_ptr(),
                                     None if sads is None else sads.data_ptr(),
                                     qmvs.data_ptr(), qsads.data_ptr()))
        return (mvs, sads), (qmvs, qsads)

    # ------------------------------------------------------- IPPP stream --
    def stream_reset(self):
        _check(lib().me_stream_reset(self._ctx))

    def stream_push(self, cf, out=None, bind_stream=True):
        """Push frame t (device or pinned host uint8 tensor [H, W]) through
        INT(t-1) || ME(t) -> SME(t) (me_stream_push).  Returns (qmvs, qsads,
        n_ref_used); outputs live where ``out`` lives (device or host)."""
        if not (isinstance(cf, torch.Tensor) and cf.dtype == torch.uint8 and cf.is_contiguous()):
            raise FevesError("cf: expected a contiguous uint8 tensor")
        on_host = not cf.is_cuda
        qmvs, qsads = out if out is not None else self.new_mvs()
        _check_out(self.mv_shape(), qmvs, qsads, "stream_push(out=)", self.device, host_ok=True)
        out_host = not qmvs.is_cuda
        n = ctypes.c_int()
        if bind_stream:
            self._bind_stream()
        _check(lib().me_stream_push(self._ctx, cf.data_ptr(), int(on_host), qmvs.data_ptr(), qsads.data_ptr(),
                                    int(out_host), ctypes.byref(n)))
        return qmvs, qsads, n.value

    def stream_push_ptr(self, cf_ptr: int, qmvs_ptr: int, qsads_ptr: int, bind_stream=True):
        """me_stream_push on raw device addresses (e.g. peer buffers mapped by
        ``ipc_open``): frame t read from ``cf_ptr``, this stripe's quarter-pel MVs /
        SADs written at ``qmvs_ptr`` / ``qsads_ptr``.  Returns n_ref_used."""
        n = ctypes.c_int()
        if bind_stream:
            self._bind_stream()
        _check(lib().me_stream_push(self._ctx, cf_ptr, 0, qmvs_ptr, qsads_ptr, 0, ctypes.byref(n)))
        return n.value

    def stream_push_flags(self, cf_ptr: int, qmvs_ptr: int, qsads_ptr: int, wait_flag: int = 0, wait_value: int = 0,
                          signal_flag: int = 0, signal_value: int = 0, bind_stream=True):
        """me_stream_push_flags on raw device addresses: the frame pull waits for
        *wait_flag >= wait_value on the copy-in stream, *signal_flag = signal_value once the
        outputs are complete (addresses 0 = none).  Returns n_ref_used."""
        n = ctypes.c_int()
        if bind_stream:
            self._bind_stream()
        _check(lib().me_stream_push_flags(self._ctx, cf_ptr, 0, qmvs_ptr, qsads_ptr, 0, ctypes.byref(n),
                                          wait_flag or None, wait_value, signal_flag or None, signal_value))
        return n.value

    def sync(self):
        _check(lib().me_sync(self._ctx))

    def stream_join(self):
        """The context (= torch current) stream waits for the internal copy / side streams
        (me_stream_join): an event recorded after this marks the end of every push so far."""
        self._bind_stream()
        _check(lib().me_stream_join(self._ctx))

    # ------------------------------------------------- peer memory (8e) --
    def ipc_export(self, t):
        """(64-byte CUDA IPC handle, byte offset) of device tensor ``t`` (me_ipc_export)."""
        h = ctypes.create_string_buffer(64)
        off = ctypes.c_size_t()
        _check(lib().me_ipc_export(self._ctx, t.data_ptr(), h, ctypes.byref(off)))
        return h.raw, off.value

    def ipc_open(self, handle: bytes, offset: int, nbytes: int) -> int:
        """Map another process's exported buffer; returns its device address (me_ipc_open)."""
        p = ctypes.c_void_p()
        _check(lib().me_ipc_open(self._ctx, ctypes.create_string_buffer(handle, 64), offset, nbytes,
                                 ctypes.byref(p)))
        return p.value

    def ipc_close(self, ptr: int):
        _check(lib().me_ipc_close(self._ctx, ptr))

    # ---------------------------------------------- module timers --
    def set_fused(self, on: bool = True):
        """SME fused into the ME kernel, or as its own launch (default)."""
        _check(lib().me_set_fused(self._ctx, int(on)))

    OPT_FUSED_SME, OPT_PIPELINE_RF, OPT_ME_CTAS_PER_SM, OPT_LAMBDA, OPT_SME_SATD, OPT_SA_INCLUSIVE = 1, 2, 3, 4, 5, 6
    OPT_HALO_ONLY, OPT_OVERLAP_SME, OPT_GRAPH, OPT_SME_KERNEL, OPT_INT_KERNEL, OPT_RF_PER_CTA = 7, 8, 9, 10, 11, 12
    OPT_SME_SPLIT = 13

    def set_sa_inclusive(self, on: bool = True):
        """Candidates in [-S/2, +S/2]^2 (G1 alternative reading, f4)."""
        self.set_option(self.OPT_SA_INCLUSIVE, int(on))

    def set_sme_satd(self, on: bool = True):
        """SME distortion = 4x4 Hadamard SATD (f4, G20) instead of SAD."""
        self.set_option(self.OPT_SME_SATD, int(on))

    def set_lambda(self, lam: int):
        """Rate term (f4, G18): ME and SME minimise SAD + lam * R(mv)."""
        self.set_option(self.OPT_LAMBDA, lam)

    def set_pmv(self, pmv):
        """MV predictor field (f4, G21; needs max_pmv > 0): int16 CUDA tensor
        [mb_rows * mb_cols, n_rf, 2] integer-pel (x, y), or None = zero predictor.
        The tensor is kept referenced: later calls read it."""
        if pmv is not None:
            if pmv.dtype != torch.int16 or not pmv.is_cuda or not pmv.is_contiguous() or \
                    pmv.numel() != self.mb_rows * self.mb_cols * self.n_rf * 2:
                raise FevesError("set_pmv: need a contiguous int16 CUDA tensor [mb_rows*mb_cols, n_rf, 2]")
        _check(lib().me_set_pmv(self._ctx, None if pmv is None else pmv.data_ptr()))
        self._pmv = pmv

    def mode_decision(self, qmvs, qsads, out=None, n_ref=None):
        """Best H.264 P-MB configuration per MB (f2, me_mode_decision) over RF slots
        [0, n_ref) (default n_rf; pass stream_push's n_ref_used on the first frames):
        int32 [rows, mb_cols, 10] = mb_type, sub_type x4, ref per 8x8 x4, cost."""
        _check_out(self.mv_shape(), qmvs, qsads, "mode_decision(qmvs, qsads)", self.device)
        shape = (self.row1 - self.row0, self.mb_cols, 10)
        o = out if out is not None else torch.empty(shape, dtype=torch.int32, device=self.device)
        if o.dtype != torch.int32 or not o.is_cuda or not o.is_contiguous() or o.numel() != shape[0] * shape[1] * 10:
            raise FevesError(f"mode_decision(out=): need a contiguous int32 CUDA tensor {shape}")
        self._bind_stream()
        _check(lib().me_mode_decision(self._ctx, qmvs.data_ptr(), qsads.data_ptr(),
                                      self.n_rf if n_ref is None else int(n_ref), o.data_ptr()))
        return o

    def set_option(self, option: int, value: int):
        """me_set_option: scheduling knobs (results identical under every setting)."""
        _check(lib().me_set_option(self._ctx, option, value))

    def set_timing(self, on: bool = True):
        _check(lib().me_set_timing(self._ctx, int(on)))

    def timings(self):
        """(ms_int, ms_me, ms_sme) of the last call; -1 for modules it did not run."""
        v = [ctypes.c_float() for _ in range(3)]
        _check(lib().me_get_timings(self._ctx, *[ctypes.byref(x) for x in v]))
        return tuple(x.value for x in v)


def stream_wait_value(stream, flag_ptr: int, value: int):
    """enqueue on a torch stream: wait until the 32-bit device word at flag_ptr >= value"""
    _check(lib().me_stream_wait_value(ctypes.c_void_p(stream.cuda_stream), flag_ptr, value))


def stream_write_value(stream, flag_ptr: int, value: int):
    """enqueue on a torch stream: write value to the 32-bit device word at flag_ptr"""
    _check(lib().me_stream_write_value(ctypes.c_void_p(stream.cuda_stream), flag_ptr, value))


__all__ = ["MotionEstimator", "FevesError", "lib", "LIB_PATH", "N_PART", "N_PHASE", "stream_wait_value",
           "stream_write_value"]
