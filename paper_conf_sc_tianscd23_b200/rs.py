"""Thin Python binding of the RSBench entry points of libxs.so (include/rs.h):
argument marshalling only.

Every step of the multipole lookup runs in the library's CUDA kernels
(csrc/rs_lookup.cu); PyTorch only owns the workspace/outputs and supplies the
current stream.  No CPU fallback: the module fails to import without
libxs.so and every call raises XSError on a library error.

Low-level functions carry the C names (``rs_init``, ``rs_workspace_size``,
``rs_lookup_batch``, ``rs_free``); ``RSProblem`` wraps them.
"""
from __future__ import annotations

import ctypes as C

from . import xs as _xs

RS_ABI_VERSION = 1
RS_FLAG_SORT, RS_FLAG_HOST_IO, RS_FLAG_BASELINE = 0x1, 0x2, 0x4

# RSBench defaults (R20): 1000 poles and 100 windows per nuclide on
# average, numL 4, doppler on, seed 42, lookup seed 1070, 10M lookups.
RS_PRESETS = {
    "rs-tiny": dict(n_nuclides=12, material_rule=1, lookups=100_000),
    "rs-small": dict(n_nuclides=68, material_rule=0, lookups=10_000_000),
    "rs-large": dict(n_nuclides=355, material_rule=0, lookups=10_000_000),
}
RS_SEED, RS_LOOKUP_SEED = 42, 1070


class rs_spec(C.Structure):
    _fields_ = [("abi_version", C.c_uint32), ("n_nuclides", C.c_int32),
                ("avg_n_poles", C.c_int32), ("avg_n_windows", C.c_int32), ("numL", C.c_int32),
                ("material_rule", C.c_int32), ("doppler", C.c_int32), ("seed", C.c_uint64),
                ("lookup_seed", C.c_uint64)]


class rs_outputs(C.Structure):
    _fields_ = [("macro_xs", C.c_void_p), ("mat", C.c_void_p), ("energy", C.c_void_p),
                ("vsum", C.c_void_p)]


def _load():
    L = _xs.lib
    P, u64, u32 = C.c_void_p, C.c_uint64, C.c_uint32
    sig = {
        "rs_init": (C.c_int, [C.POINTER(rs_spec), C.c_int, P, C.POINTER(P)]),
        "rs_workspace_size": (C.c_int, [P, u64, u32, C.POINTER(C.c_size_t)]),
        "rs_lookup_batch": (C.c_int, [P, u64, u64, u32, C.POINTER(rs_outputs), P, C.c_size_t,
                                      P]),
        "rs_lookup_explicit": (C.c_int, [P, P, P, u64, u32, C.POINTER(rs_outputs), P,
                                         C.c_size_t, P]),
        "rs_work_count": (C.c_int, [P, u64, u64, P, P]),
        "rs_set_param": (C.c_int, [P, C.c_char_p, C.c_int64]),
        "rs_launch_count": (u64, [P]),
        "rs_device_bytes": (u64, [P]),
        "rs_free": (None, [P]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    return L


lib = _load()
_check = _xs._check


def rs_init(spec: rs_spec, device: int, stream: int) -> int:
    h = C.c_void_p()
    _check(lib.rs_init(C.byref(spec), device, C.c_void_p(stream), C.byref(h)))
    return h.value


def rs_workspace_size(d: int, count: int, flags: int) -> int:
    n = C.c_size_t()
    _check(lib.rs_workspace_size(d, count, flags, C.byref(n)))
    return n.value


def rs_lookup_batch(d, first_id, count, flags, out: rs_outputs, workspace, ws_bytes, stream):
    _check(lib.rs_lookup_batch(d, first_id, count, flags, C.byref(out), workspace, ws_bytes,
                               C.c_void_p(stream)))


def rs_lookup_explicit(d, energy, mat, count, flags, out: rs_outputs, workspace, ws_bytes, stream):
    _check(lib.rs_lookup_explicit(d, energy, mat, count, flags, C.byref(out), workspace, ws_bytes,
                                  C.c_void_p(stream)))


def rs_work_count(d, first_id, count, work, stream):
    _check(lib.rs_work_count(d, first_id, count, work, C.c_void_p(stream)))


def rs_set_param(d, name: str, value: int):
    _check(lib.rs_set_param(d, name.encode(), value))


def rs_launch_count(d) -> int:
    return lib.rs_launch_count(d)


def rs_device_bytes(d) -> int:
    return lib.rs_device_bytes(d)


def rs_free(d):
    lib.rs_free(d)


def make_spec(n_nuclides=355, avg_n_poles=1000, avg_n_windows=100, numL=4, material_rule=0,
              doppler=1, seed=RS_SEED, lookup_seed=RS_LOOKUP_SEED, **_):
    return rs_spec(RS_ABI_VERSION, n_nuclides, avg_n_poles, avg_n_windows, numL, material_rule,
                   doppler, seed, lookup_seed)


class RSProblem:
    """One replica of the RSBench tables on one CUDA device."""

    def __init__(self, handle: int, device: int):
        import torch
        self._h = handle
        self.device = torch.device("cuda", device)
        self._ws = None

    @classmethod
    def from_spec(cls, device: int = 0, **spec_kw):
        import torch
        with torch.cuda.device(device):
            st = torch.cuda.current_stream().cuda_stream
            return cls(rs_init(make_spec(**spec_kw), device, st), device)

    @classmethod
    def from_preset(cls, name: str, device: int = 0, **over):
        kw = dict(RS_PRESETS[name])
        kw.update(over)
        return cls.from_spec(device=device, **kw)

    def close(self):
        h, self._h = getattr(self, "_h", None), None
        if h:
            rs_free(h)

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_param(self, name: str, value: int):
        rs_set_param(self._h, name, value)

    @property
    def launches(self) -> int:
        return rs_launch_count(self._h)

    @property
    def device_bytes(self) -> int:
        return rs_device_bytes(self._h)

    def work_count(self, first_id: int, count: int):
        """(lookup-nuclide evaluations, pole terms) of a batch (instrumentation)."""
        import torch
        w = torch.zeros(2, dtype=torch.int64, device=self.device)
        rs_work_count(self._h, first_id, count, w.data_ptr(),
                      torch.cuda.current_stream(self.device).cuda_stream)
        return [int(x) for x in w.cpu()]

    def workspace(self, count: int, flags: int = 0):
        import torch
        n = rs_workspace_size(self._h, count, flags)
        if self._ws is None or self._ws.numel() < n:
            self._ws = torch.empty(max(n, 256), dtype=torch.uint8, device=self.device)
        return self._ws

    def lookup(self, first_id: int, count: int, sort: bool = True, baseline: bool = False,
               want=(), vsum=None):
        """R1-R7 for lookup ids [first_id, first_id+count) on the current stream.
        Returns (vsum tensor [2] on device, dict of the outputs in `want`:
        macro_xs [count][4], mat, energy)."""
        import torch
        flags = (RS_FLAG_SORT if sort else 0) | (RS_FLAG_BASELINE if baseline else 0)
        if vsum is None:
            vsum = torch.zeros(2, dtype=torch.int64, device=self.device)
        res = {}

        def mk(name, shape, dt):
            if name in want:
                t = torch.empty(shape, dtype=dt, device=self.device)
                res[name] = t
                return t.data_ptr()
            return None
        o = rs_outputs(mk("macro_xs", (count, 4), torch.float64),
                       mk("mat", (count,), torch.int32), mk("energy", (count,), torch.float64),
                       vsum.data_ptr())
        ws = self.workspace(count, flags)
        st = torch.cuda.current_stream(self.device).cuda_stream  # torch's allocator orders reuse here
        rs_lookup_batch(self._h, first_id, count, flags, o, ws.data_ptr(), ws.numel(), st)
        return vsum, res

    def lookup_explicit(self, energy, mat, sort: bool = True, want=(), vsum=None):
        """R2-R7 for caller-given energies (float64) and materials (uint8).
        CUDA tensors, or CPU tensors (then RS_FLAG_HOST_IO: staged copies inside
        the call, which synchronizes; only macro_xs may be requested)."""
        import torch
        host = not energy.is_cuda
        assert mat.dtype == torch.uint8 and energy.dtype == torch.float64
        count = energy.numel()
        flags = (RS_FLAG_SORT if sort else 0) | (RS_FLAG_HOST_IO if host else 0)
        dev = "cpu" if host else self.device
        if vsum is None:
            vsum = torch.zeros(2, dtype=torch.int64, device=dev)
        res = {}

        def mk(name, shape, dt):
            if name in want:
                t = torch.empty(shape, dtype=dt, device=dev,
                                pin_memory=host and torch.cuda.is_available())
                res[name] = t
                return t.data_ptr()
            return None
        o = rs_outputs(mk("macro_xs", (count, 4), torch.float64),
                       mk("mat", (count,), torch.int32), mk("energy", (count,), torch.float64),
                       vsum.data_ptr())
        ws = self.workspace(count, flags)
        st = torch.cuda.current_stream(self.device).cuda_stream  # torch's allocator orders reuse here
        rs_lookup_explicit(self._h, energy.data_ptr(), mat.data_ptr(), count, flags, o,
                           ws.data_ptr(), ws.numel(), st)
        return vsum, res
