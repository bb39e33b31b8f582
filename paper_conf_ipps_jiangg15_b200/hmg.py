"""Thin ctypes binding of libhmg (include/hmg.h): argument marshalling only.

Every step of the path runs in libhmg's CUDA kernels; this module converts
numpy / torch arguments to pointers and maps status codes to exceptions.
PyTorch supplies device memory (output tensors) and streams.  There is no CPU
fallback: if libhmg.so is missing or no CUDA device is present the calls raise.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIBPATH = os.path.join(_HERE, "libhmg.so")
_lib = None

HMG_OK, HMG_EINVAL, HMG_ENOMEM, HMG_ECUDA, HMG_EUNSUPPORTED = range(5)

c_int, c_i64, c_f, c_d, c_p = ctypes.c_int, ctypes.c_int64, ctypes.c_float, ctypes.c_double, ctypes.c_void_p


class hmg_evparams(ctypes.Structure):
    _fields_ = [("mu_msv", c_d), ("lambda_msv", c_d), ("mu_vit", c_d), ("lambda_vit", c_d)]


class hmg_quant(ctypes.Structure):
    _fields_ = [("M", c_int), ("bias_b", c_int), ("tbm_b", c_int), ("tec_b", c_int), ("base_b", c_int),
                ("scale_b", c_f), ("base_w", c_int), ("xw_e", c_int), ("ddbound_w", c_int), ("scale_w", c_f),
                ("cost", ctypes.POINTER(ctypes.c_uint8)), ("rsc", ctypes.POINTER(ctypes.c_int16)),
                ("tsc", ctypes.POINTER(ctypes.c_int16)), ("msv_fast", c_int), ("msv_lanes", c_int),
                ("msv_regs", c_int), ("vit_lanes", c_int), ("vit_nodes", c_int),
                ("vit_pair_lanes", c_int), ("vit_pair_regs", c_int),
                ("fwd_warps", c_int), ("fwd_nodes", c_int), ("fwd_rows_smem", c_int),
                ("fwd_seqs_per_block", c_int), ("fwd_lanes", c_int), ("vit_pair_kernel", c_int)]


# name -> (restype, argtypes), exactly the declarations of include/hmg.h
SIGNATURES = {
    "hmg_profile_create": (c_int, [c_int, c_p, c_p, c_p, c_int, ctypes.POINTER(c_p)]),
    "hmg_profile_quant": (c_int, [c_p, ctypes.POINTER(hmg_quant)]),
    "hmg_profile_destroy": (None, [c_p]),
    "hmg_db_create": (c_int, [c_p, c_p, c_i64, c_int, ctypes.POINTER(c_p)]),
    "hmg_db_nseq": (c_i64, [c_p]),
    "hmg_db_residues": (c_i64, [c_p]),
    "hmg_db_packed_bytes": (c_i64, [c_p]),
    "hmg_db_long_lane": (c_i64, [c_p, c_p]),
    "hmg_db_order": (c_int, [c_p, c_p]),
    "hmg_db_image": (c_int, [c_p, c_p]),
    "hmg_db_upload": (c_int, [c_p, c_p, c_p]),
    "hmg_db_destroy": (None, [c_p]),
    "hmg_msv": (c_int, [c_p, c_p, c_d, c_p, c_p, c_p]),
    "hmg_viterbi": (c_int, [c_p, c_p, c_p, c_i64, c_d, c_p, c_p, c_p]),
    "hmg_pipeline": (c_int, [c_p, c_p, c_d, c_d, c_p, c_p, c_p, c_p, c_p, c_p]),
    "hmg_pipeline_upload": (c_int, [c_p, c_p, c_p, c_d, c_d, c_p, c_p, c_p, c_p, c_p, c_p]),
    "hmg_forward": (c_int, [c_p, c_p, c_p, c_i64, c_p, c_p]),
    "hmg_pipeline_forward": (c_int, [c_p, c_p, c_d, c_d, c_p, c_p, c_p, c_p, c_p, c_p, c_p, c_p, c_p]),
    "hmg_msv_batch": (c_int, [c_p, c_int, c_p, c_d, c_p, c_p, c_p]),
    "hmg_pipeline_batch": (c_int, [c_p, c_int, c_p, c_d, c_d, c_p, c_p, c_p, c_p, c_p, c_p, c_p, c_p, c_p]),
    "hmg_msv_nats": (c_f, [c_int, c_int]),
    "hmg_vit_nats": (c_f, [c_int, c_int]),
    "hmg_null1_nats": (c_f, [c_int]),
    "hmg_gumbel_surv": (c_d, [c_d, c_d, c_d]),
    "hmg_strerror": (ctypes.c_char_p, [c_int]),
    "hmg_kernel_launches": (c_i64, []),
    "hmg_calibrate": (c_int, [c_p, c_int, c_int, ctypes.c_uint64, c_d, c_p]),
    "hmg_calibrate_db": (c_int, [c_p, c_p, c_d, c_p]),
    "hmg_prepare_thresholds": (c_int, [c_p, c_d, c_d, c_int]),
    "hmg_set_tuning": (c_int, [ctypes.c_char_p, c_int]),
    "hmg_clear_tuning": (c_int, [ctypes.c_char_p]),
    "hmg_set_stage_timing": (c_int, [c_int]),
    "hmg_stage_times": (c_int, [c_p]),
    "hmg_stage_counts": (c_int, [c_p]),
}


class HmgError(RuntimeError):
    def __init__(self, status, what):
        super().__init__("%s: %s (status %d)" % (what, lib().hmg_strerror(status).decode(), status))
        self.status = status


def lib():
    """Load libhmg.so (built by paper_conf_ipps_jiangg15_b200.build); raises if absent."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIBPATH):
            raise RuntimeError("libhmg.so not built (run python -m paper_conf_ipps_jiangg15_b200.build); "
                               "there is no CPU fallback")
        L = ctypes.CDLL(LIBPATH)
        for name, (res, args) in SIGNATURES.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _check(st, what):
    if st != HMG_OK:
        raise HmgError(st, what)


def _np_ptr(a):
    return a.ctypes.data_as(c_p) if a is not None else None


def _dev_ptr(t):
    """Device pointer of a CUDA torch tensor (must be contiguous)."""
    if t is None:
        return None
    if not t.is_cuda:
        raise ValueError("expected a CUDA tensor")
    if not t.is_contiguous():
        raise ValueError("expected a contiguous tensor")
    return c_p(t.data_ptr())


def _stream_ptr(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return c_p(stream.cuda_stream)


# ------------------------------------------------------------------------ profile
class Profile:
    """hmg_profile: a quantised profile resident on one device."""

    def __init__(self, msc, tsc=None, ev=None, device: int = 0):
        msc = np.ascontiguousarray(msc, dtype=np.float32)
        self.M = msc.shape[0]
        if msc.shape != (self.M, 29):
            raise ValueError("msc must be [M][29]")
        if tsc is not None:
            tsc = np.ascontiguousarray(tsc, dtype=np.float32)
            if tsc.shape != (self.M, 8):
                raise ValueError("tsc must be [M][8]")
        evp = None
        if ev is not None:
            evp = hmg_evparams(*[float(v) for v in ev])
        h = c_p()
        _check(lib().hmg_profile_create(self.M, _np_ptr(msc), _np_ptr(tsc),
                                        ctypes.byref(evp) if evp is not None else None, device, ctypes.byref(h)),
               "hmg_profile_create")
        self._h = h
        self._destroy = lib().hmg_profile_destroy
        self.device = device

    @property
    def handle(self):
        return self._h

    def quant(self) -> dict:
        q = hmg_quant()
        _check(lib().hmg_profile_quant(self._h, ctypes.byref(q)), "hmg_profile_quant")
        M = q.M
        d = {k: getattr(q, k) for k, _ in hmg_quant._fields_ if k not in ("cost", "rsc", "tsc")}
        d["cost"] = np.ctypeslib.as_array(q.cost, shape=(29 * M,)).reshape(29, M).copy()
        d["rsc"] = np.ctypeslib.as_array(q.rsc, shape=(29 * M,)).reshape(29, M).copy()
        d["tsc"] = (np.ctypeslib.as_array(q.tsc, shape=(8 * M,)).reshape(8, M).copy() if q.tsc else None)
        return d

    def calibrate(self, n: int = 1000, L: int = 200, seed: int = 7, lam: float = 0.6931471805599453):
        """Gumbel (mu_msv, lambda, mu_vit, lambda) fitted on the GPU (hmg_calibrate)."""
        ev = hmg_evparams()
        _check(lib().hmg_calibrate(self._h, n, L, seed, lam, ctypes.byref(ev)), "hmg_calibrate")
        return (ev.mu_msv, ev.lambda_msv, ev.mu_vit, ev.lambda_vit)

    def calibrate_db(self, db, lam: float = 0.6931471805599453):
        """Gumbel (mu_msv, lambda, mu_vit, lambda) fitted on the GPU scores of ``db`` (hmg_calibrate_db)."""
        ev = hmg_evparams()
        _check(lib().hmg_calibrate_db(self._h, db.handle, lam, ctypes.byref(ev)), "hmg_calibrate_db")
        return (ev.mu_msv, ev.lambda_msv, ev.mu_vit, ev.lambda_vit)

    def close(self):
        if getattr(self, "_h", None):
            self._destroy(self._h)
            self._h = None

    __del__ = close


# ------------------------------------------------------------------------ database
class Database:
    """hmg_db: a packed, length-sorted DB (shard) resident on one device."""

    def __init__(self, dsq, off, device: int = 0):
        dsq = np.ascontiguousarray(dsq, dtype=np.uint8)
        off = np.ascontiguousarray(off, dtype=np.int64)
        self.nseq = len(off) - 1
        h = c_p()
        _check(lib().hmg_db_create(_np_ptr(dsq) if len(dsq) else None, _np_ptr(off), self.nseq, device,
                                   ctypes.byref(h)), "hmg_db_create")
        self._h = h
        self._destroy = lib().hmg_db_destroy
        self.device = device
        self.lengths = np.diff(off).astype(np.int32)

    @property
    def handle(self):
        return self._h

    @property
    def residues(self) -> int:
        return lib().hmg_db_residues(self._h)

    @property
    def packed_bytes(self) -> int:
        return lib().hmg_db_packed_bytes(self._h)

    def long_lane(self):
        """(number of long-lane sequences, their residues) -- DESIGN.md 4.4."""
        r = ctypes.c_int64()
        n = lib().hmg_db_long_lane(self._h, ctypes.byref(r))
        return int(n), int(r.value)

    def order(self) -> np.ndarray:
        o = np.zeros(self.nseq, dtype=np.int32)
        _check(lib().hmg_db_order(self._h, _np_ptr(o)), "hmg_db_order")
        return o

    def image(self, out=None):
        """Packed residue image into a host buffer (numpy uint32 or pinned torch tensor)."""
        n = self.packed_bytes // 4
        if out is None:
            out = np.zeros(n, dtype=np.uint32)
            _check(lib().hmg_db_image(self._h, _np_ptr(out)), "hmg_db_image")
        else:
            _check(lib().hmg_db_image(self._h, c_p(out.data_ptr())), "hmg_db_image")
        return out

    def upload(self, image, stream=None):
        """Asynchronous H2D re-upload of a packed image held in (pinned) host memory."""
        ptr = c_p(image.data_ptr()) if hasattr(image, "data_ptr") else _np_ptr(image)
        _check(lib().hmg_db_upload(self._h, ptr, _stream_ptr(stream)), "hmg_db_upload")

    def close(self):
        if getattr(self, "_h", None):
            self._destroy(self._h)
            self._h = None

    __del__ = close


# ------------------------------------------------------------------------ filters
def hmg_msv(profile: Profile, db: Database, raw, pass_=None, F1: float = 0.02, stream=None):
    """MSV filter (Alg 1) into device tensors raw (uint8 [nseq]) and pass_ (uint8 or None)."""
    _check(lib().hmg_msv(profile.handle, db.handle, F1, _stream_ptr(stream), _dev_ptr(raw), _dev_ptr(pass_)),
           "hmg_msv")


def hmg_viterbi(profile: Profile, db: Database, raw, ids=None, pass_=None, F2: float = 1e-3, stream=None):
    """Viterbi filter (Alg 2) over device int32 ``ids`` (caller order; None = all)."""
    n = 0 if ids is None else int(ids.numel())
    _check(lib().hmg_viterbi(profile.handle, db.handle, _dev_ptr(ids), n, F2, _stream_ptr(stream),
                             _dev_ptr(raw), _dev_ptr(pass_)), "hmg_viterbi")


def hmg_pipeline(profile: Profile, db: Database, msv_raw, vit_raw, flags, survivor_ids, n_survivors,
                 F1: float = 0.02, F2: float = 1e-3, stream=None):
    """MSV -> pass flags -> device compaction -> Viterbi over survivors (Fig 1)."""
    _check(lib().hmg_pipeline(profile.handle, db.handle, F1, F2, _stream_ptr(stream), _dev_ptr(msv_raw),
                              _dev_ptr(vit_raw), _dev_ptr(flags), _dev_ptr(survivor_ids),
                              _dev_ptr(n_survivors)), "hmg_pipeline")


def hmg_forward(profile: Profile, db: Database, nats, ids=None, stream=None):
    """Forward stage (f2; Fig 1) over device int32 ``ids`` (caller order; None = all)
    into the device float32 tensor ``nats`` [nseq]."""
    n = 0 if ids is None else int(ids.numel())
    _check(lib().hmg_forward(profile.handle, db.handle, _dev_ptr(ids), n, _stream_ptr(stream), _dev_ptr(nats)),
           "hmg_forward")


def hmg_pipeline_forward(profile: Profile, db: Database, msv_raw, vit_raw, flags, survivor_ids, n_survivors,
                         fwd_nats, fwd_ids, n_fwd, F1: float = 0.02, F2: float = 1e-3, stream=None):
    """MSV -> compaction -> Viterbi -> compaction of the Viterbi passes -> Forward (Fig 1)."""
    _check(lib().hmg_pipeline_forward(profile.handle, db.handle, F1, F2, _stream_ptr(stream), _dev_ptr(msv_raw),
                                      _dev_ptr(vit_raw), _dev_ptr(flags), _dev_ptr(survivor_ids),
                                      _dev_ptr(n_survivors), _dev_ptr(fwd_nats), _dev_ptr(fwd_ids),
                                      _dev_ptr(n_fwd)), "hmg_pipeline_forward")


def hmg_msv_batch(profiles, db: Database, raw, pass_=None, F1: float = 0.02, stream=None):
    """Many-profile MSV (f4): raw (uint8 [nprof][nseq]) and pass_ for every (profile, sequence) pair."""
    arr = (c_p * len(profiles))(*[p.handle for p in profiles])
    _check(lib().hmg_msv_batch(arr, len(profiles), db.handle, F1, _stream_ptr(stream), _dev_ptr(raw),
                               _dev_ptr(pass_)), "hmg_msv_batch")


def hmg_pipeline_batch(profiles, db: Database, msv_raw, vit_raw, flags, survivor_ids, n_survivors,
                       F1: float = 0.02, F2: float = 1e-3, stream=None, fwd_nats=None, fwd_ids=None, n_fwd=None):
    """Fig 1 filter pipeline for every profile of a batch (f4); outputs are [nprof][nseq] rows;
    with fwd_nats / fwd_ids / n_fwd also the Forward stage on each profile's Viterbi passes."""
    arr = (c_p * len(profiles))(*[p.handle for p in profiles])
    _check(lib().hmg_pipeline_batch(arr, len(profiles), db.handle, F1, F2, _stream_ptr(stream), _dev_ptr(msv_raw),
                                    _dev_ptr(vit_raw), _dev_ptr(flags), _dev_ptr(survivor_ids),
                                    _dev_ptr(n_survivors), _dev_ptr(fwd_nats), _dev_ptr(fwd_ids),
                                    _dev_ptr(n_fwd)), "hmg_pipeline_batch")


def alloc_batch_outputs(nprof: int, nseq: int, device: int = 0):
    """Caller-owned device outputs for hmg_pipeline_batch."""
    import torch
    dev = torch.device("cuda", device)
    return dict(msv_raw=torch.zeros((nprof, nseq), dtype=torch.uint8, device=dev),
                vit_raw=torch.full((nprof, nseq), -32768, dtype=torch.int16, device=dev),
                flags=torch.zeros((nprof, nseq), dtype=torch.uint8, device=dev),
                survivor_ids=torch.zeros((nprof, max(nseq, 1)), dtype=torch.int32, device=dev),
                n_survivors=torch.zeros(nprof, dtype=torch.int64, device=dev))


def alloc_batch_forward_outputs(nprof: int, nseq: int, device: int = 0):
    """Optional Forward outputs of hmg_pipeline_batch."""
    import torch
    dev = torch.device("cuda", device)
    return dict(fwd_nats=torch.full((nprof, nseq), float("nan"), dtype=torch.float32, device=dev),
                fwd_ids=torch.zeros((nprof, max(nseq, 1)), dtype=torch.int32, device=dev),
                n_fwd=torch.zeros(nprof, dtype=torch.int64, device=dev))


def hmg_pipeline_upload(profile: Profile, db: Database, image, msv_raw, vit_raw, flags, survivor_ids, n_survivors,
                        F1: float = 0.02, F2: float = 1e-3, stream=None):
    """Upload of the packed image (pinned host tensor from Database.image) overlapped with the
    pipeline: MSV scores each length-ordered part as it lands (hmg_pipeline_upload)."""
    ptr = c_p(image.data_ptr()) if hasattr(image, "data_ptr") else _np_ptr(image)
    _check(lib().hmg_pipeline_upload(profile.handle, db.handle, ptr, F1, F2, _stream_ptr(stream),
                                     _dev_ptr(msv_raw), _dev_ptr(vit_raw), _dev_ptr(flags),
                                     _dev_ptr(survivor_ids), _dev_ptr(n_survivors)), "hmg_pipeline_upload")


def hmg_msv_nats(raw: int, L: int) -> float:
    return lib().hmg_msv_nats(int(raw), int(L))


def hmg_vit_nats(raw: int, L: int) -> float:
    return lib().hmg_vit_nats(int(raw), int(L))


def hmg_null1_nats(L: int) -> float:
    return lib().hmg_null1_nats(int(L))


def hmg_gumbel_surv(bits: float, mu: float, lam: float) -> float:
    return lib().hmg_gumbel_surv(bits, mu, lam)


STAGES = ("msv_kernel", "msv_redo", "msv_flags_compaction", "vit_kernel", "vit_flags", "fwd")


def hmg_kernel_launches() -> int:
    return lib().hmg_kernel_launches()


def hmg_set_stage_timing(enable: bool = True):
    _check(lib().hmg_set_stage_timing(int(enable)), "hmg_set_stage_timing")


def hmg_stage_times() -> dict:
    ms = np.zeros(len(STAGES), dtype=np.float64)
    _check(lib().hmg_stage_times(_np_ptr(ms)), "hmg_stage_times")
    return dict(zip(STAGES, ms.tolist()))


def hmg_stage_counts() -> dict:
    """Counts of the most recent call (stage timing on): sequences the s16x2 pair Viterbi kernel
    handed back to the s32 kernel (-1: the pair kernel did not run)."""
    c = np.zeros(1, dtype=np.int64)
    _check(lib().hmg_stage_counts(_np_ptr(c)), "hmg_stage_counts")
    return {"vit_pair_redo": int(c[0])}


def hmg_prepare_thresholds(profile: Profile, F1: float = 0.02, F2: float = 1e-3, Lmax: int = 40000):
    _check(lib().hmg_prepare_thresholds(profile.handle, F1, F2, Lmax), "hmg_prepare_thresholds")


def set_tuning(name: str, value: int):
    """Performance knob override (hmg_set_tuning); results never depend on it."""
    _check(lib().hmg_set_tuning(name.encode(), int(value)), "hmg_set_tuning(%s)" % name)


def clear_tuning(name: str | None = None):
    _check(lib().hmg_clear_tuning(name.encode() if name else None), "hmg_clear_tuning")


class tuning:
    """with hmg.tuning(VIT_PAIR_W=4): ... -- overrides for the block, cleared after."""

    def __init__(self, **kw):
        self.kw = kw

    def __enter__(self):
        for k, v in self.kw.items():
            set_tuning(k, v)
        return self

    def __exit__(self, *a):
        for k in self.kw:
            clear_tuning(k)


# ------------------------------------------------------------------------ convenience
def calibrated_profile(msc, tsc, device: int = 0, n: int = 1000, L: int = 200, seed: int = 7):
    """A profile with its Gumbel locations fitted on the GPU (hmg_calibrate, lambda = ln 2,
    P:41-45): profiles are immutable, so the searching profile is created with the fit."""
    p = Profile(msc, tsc, device=device)
    ev = p.calibrate(n=n, L=L, seed=seed)
    p.close()
    return Profile(msc, tsc, ev=ev, device=device), ev


def alloc_outputs(nseq: int, device: int = 0):
    """Caller-owned device outputs for hmg_pipeline (torch provides the memory)."""
    import torch
    dev = torch.device("cuda", device)
    return dict(msv_raw=torch.zeros(nseq, dtype=torch.uint8, device=dev),
                vit_raw=torch.full((nseq,), -32768, dtype=torch.int16, device=dev),
                flags=torch.zeros(nseq, dtype=torch.uint8, device=dev),
                survivor_ids=torch.zeros(max(nseq, 1), dtype=torch.int32, device=dev),
                n_survivors=torch.zeros(1, dtype=torch.int64, device=dev))


def alloc_forward_outputs(nseq: int, device: int = 0):
    """Extra caller-owned device outputs of hmg_pipeline_forward."""
    import torch
    dev = torch.device("cuda", device)
    return dict(fwd_nats=torch.full((nseq,), float("nan"), dtype=torch.float32, device=dev),
                fwd_ids=torch.zeros(max(nseq, 1), dtype=torch.int32, device=dev),
                n_fwd=torch.zeros(1, dtype=torch.int64, device=dev))
