"""Thin Python binding of libxs.so (include/xs.h): argument marshalling only.

Every step of the lookup path runs in the library's CUDA kernels; PyTorch is
used here only to own device memory (workspace, outputs) and to supply the
current CUDA stream.  There is no CPU fallback: importing this module fails
loudly when libxs.so is missing, and every call raises XSError when the
library reports an error.

The low-level functions carry the C names (``xs_init_grid``,
``xs_lookup_batch``, ``xs_lookup_explicit``, ``xs_verify``, ...); ``Grid`` is a
convenience wrapper over them.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libxs.so")

XS_ABI_VERSION = 1
XS_GRID_UNIONIZED, XS_GRID_NUCLIDE, XS_GRID_HASH = 0, 1, 2
XS_FLAG_SORT, XS_FLAG_HOST_IO, XS_FLAG_BASELINE, XS_FLAG_F32 = 0x1, 0x2, 0x4, 0x8
XS_FLAG_MAT_U8 = 0x10
XS_FLAG_HOST_ASYNC = 0x20
(XS_TABLE_NUCLIDE_GRID, XS_TABLE_UNION_ENERGY, XS_TABLE_INDEX_GRID, XS_TABLE_NUM_NUCS,
 XS_TABLE_MATS, XS_TABLE_CONCS, XS_TABLE_INDEX_GRID_T, XS_TABLE_INTERVALS,
 XS_TABLE_INTERVALS32, XS_TABLE_INTERVALS_U) = range(10)
XS_INDEX_AUTO, XS_INDEX_ROW, XS_INDEX_COL, XS_INDEX_BOTH = 0, 1, 2, 3
INDEX_LAYOUTS = {"auto": 0, "row": 1, "col": 2, "both": 3}
STATUS = {0: "XS_OK", 1: "XS_ERR_INVALID_ARG", 2: "XS_ERR_OUT_OF_MEMORY", 3: "XS_ERR_CUDA",
          4: "XS_ERR_UNSUPPORTED", 5: "XS_ERR_STATE", 6: "XS_ERR_DATA"}
GRID_TYPES = {"unionized": XS_GRID_UNIONIZED, "nuclide": XS_GRID_NUCLIDE, "hash": XS_GRID_HASH}


class XSError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class xs_grid_spec(C.Structure):
    _fields_ = [("abi_version", C.c_uint32), ("n_isotopes", C.c_int32),
                ("n_gridpoints", C.c_int64), ("grid_type", C.c_int32), ("hash_bins", C.c_int32),
                ("grid_seed", C.c_uint64), ("conc_seed", C.c_uint64), ("lookup_seed", C.c_uint64),
                ("material_rule", C.c_int32), ("index_layout", C.c_int32)]


class xs_grid_data(C.Structure):
    _fields_ = [("abi_version", C.c_uint32), ("n_isotopes", C.c_int32),
                ("n_gridpoints", C.c_int64), ("nuclide_grid", C.c_void_p),
                ("n_mats", C.c_int32), ("max_num_nucs", C.c_int32), ("num_nucs", C.c_void_p),
                ("mats", C.c_void_p), ("concs", C.c_void_p), ("grid_type", C.c_int32),
                ("hash_bins", C.c_int32), ("lookup_seed", C.c_uint64),
                ("index_layout", C.c_int32), ("reserved0", C.c_int32)]


class xs_grid_info(C.Structure):
    _fields_ = [("n_isotopes", C.c_int32), ("n_mats", C.c_int32), ("max_num_nucs", C.c_int32),
                ("grid_type", C.c_int32), ("hash_bins", C.c_int32), ("device", C.c_int32),
                ("n_gridpoints", C.c_int64), ("n_union", C.c_int64),
                ("index_grid_len", C.c_int64), ("device_bytes", C.c_uint64),
                ("lookup_seed", C.c_uint64), ("index_layout", C.c_int32),
                ("reserved0", C.c_int32)]


class xs_timing(C.Structure):
    _fields_ = [("calls", C.c_uint64), ("kernel_launches", C.c_uint64),
                ("ms_count", C.c_double), ("ms_bucket", C.c_double), ("ms_gather", C.c_double),
                ("ms_total", C.c_double)]


class xs_outputs(C.Structure):
    _fields_ = [("macro_xs", C.c_void_p), ("energy", C.c_void_p), ("mat", C.c_void_p),
                ("grid_index", C.c_void_p), ("verification", C.c_void_p), ("vsum", C.c_void_p)]


EXPORTS = ["xs_abi_version", "xs_init_grid", "xs_init_grid_data", "xs_grid_get_info",
           "xs_workspace_size", "xs_lookup_batch", "xs_lookup_explicit", "xs_verify",
           "xs_nuclide_index", "xs_get_table", "xs_set_param", "xs_hash_finalize",
           "xs_free_grid", "xs_last_error", "xs_timing_enable", "xs_timing_read",
           "xs_history_workspace_size", "xs_lookup_history", "xs_lookup_batch_shard"]


def _load() -> C.CDLL:
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"libxs.so not built ({LIB_PATH}); run "
                          "`python -m paper_conf_sc_tianscd23_b200.build` — there is no CPU "
                          "fallback for the lookup path")
    L = C.CDLL(LIB_PATH)
    P, u64, i64, i32, u32 = C.c_void_p, C.c_uint64, C.c_int64, C.c_int32, C.c_uint32
    st = C.c_int
    sig = {
        "xs_abi_version": (u32, []),
        "xs_init_grid": (st, [C.POINTER(xs_grid_spec), C.c_int, P, C.POINTER(P)]),
        "xs_init_grid_data": (st, [C.POINTER(xs_grid_data), C.c_int, P, C.POINTER(P)]),
        "xs_grid_get_info": (st, [P, C.POINTER(xs_grid_info)]),
        "xs_workspace_size": (st, [P, u64, u32, C.POINTER(C.c_size_t)]),
        "xs_lookup_batch": (st, [P, u64, u64, u32, C.POINTER(xs_outputs), P, C.c_size_t, P]),
        "xs_lookup_explicit": (st, [P, P, P, u64, u32, C.POINTER(xs_outputs), P, C.c_size_t, P]),
        "xs_lookup_batch_shard": (st, [P, u64, u64, i32, i32, u32, C.POINTER(xs_outputs), P,
                                       C.c_size_t, P]),
        "xs_verify": (st, [P, P, u64, P, P]),
        "xs_nuclide_index": (st, [P, P, P, u64, P, P]),
        "xs_get_table": (st, [P, i32, u64, u64, P]),
        "xs_set_param": (st, [P, C.c_char_p, i64]),
        "xs_hash_finalize": (u64, [u64]),
        "xs_free_grid": (None, [P]),
        "xs_last_error": (C.c_char_p, []),
        "xs_timing_enable": (st, [P, C.c_int]),
        "xs_timing_read": (st, [P, C.POINTER(xs_timing)]),
        "xs_history_workspace_size": (st, [P, u64, u32, C.POINTER(C.c_size_t)]),
        "xs_lookup_history": (st, [P, u64, u64, i32, u32, C.POINTER(xs_outputs), P, C.c_size_t,
                                   P]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    if L.xs_abi_version() != XS_ABI_VERSION:
        raise ImportError("libxs.so ABI version mismatch")
    return L


lib = _load()


def _check(status: int):
    if status != 0:
        raise XSError(status, lib.xs_last_error().decode(errors="replace"))


# ------------------------------------------------------- C-named functions
def xs_abi_version() -> int:
    return lib.xs_abi_version()


def xs_init_grid(spec: xs_grid_spec, device: int, stream: int) -> int:
    h = C.c_void_p()
    _check(lib.xs_init_grid(C.byref(spec), device, stream, C.byref(h)))
    return h.value


def xs_init_grid_data(data: xs_grid_data, device: int, stream: int) -> int:
    h = C.c_void_p()
    _check(lib.xs_init_grid_data(C.byref(data), device, stream, C.byref(h)))
    return h.value


def xs_grid_get_info(g: int) -> xs_grid_info:
    info = xs_grid_info()
    _check(lib.xs_grid_get_info(g, C.byref(info)))
    return info


def xs_workspace_size(g: int, count: int, flags: int) -> int:
    n = C.c_size_t()
    _check(lib.xs_workspace_size(g, count, flags, C.byref(n)))
    return n.value


def xs_lookup_batch(g, first_id, count, flags, out: xs_outputs, workspace, ws_bytes, stream):
    _check(lib.xs_lookup_batch(g, first_id, count, flags, C.byref(out), workspace, ws_bytes,
                               stream))


def xs_lookup_batch_shard(g, first_id, count, shard, n_shards, flags, out: xs_outputs, workspace,
                          ws_bytes, stream):
    _check(lib.xs_lookup_batch_shard(g, first_id, count, shard, n_shards, flags, C.byref(out),
                                     workspace, ws_bytes, stream))


def xs_lookup_explicit(g, energy, mat, count, flags, out: xs_outputs, workspace, ws_bytes,
                       stream):
    _check(lib.xs_lookup_explicit(g, energy, mat, count, flags, C.byref(out), workspace,
                                  ws_bytes, stream))


def xs_history_workspace_size(g: int, n_particles: int, flags: int) -> int:
    n = C.c_size_t()
    _check(lib.xs_history_workspace_size(g, n_particles, flags, C.byref(n)))
    return n.value


def xs_lookup_history(g, first_particle, n_particles, lookups, flags, out: xs_outputs, workspace,
                      ws_bytes, stream):
    _check(lib.xs_lookup_history(g, first_particle, n_particles, lookups, flags, C.byref(out),
                                 workspace, ws_bytes, stream))


def xs_verify(g, macro_xs, count, vsum, stream):
    _check(lib.xs_verify(g, macro_xs, count, vsum, stream))


def xs_nuclide_index(g, energy, nuclide, count, k_out, stream):
    _check(lib.xs_nuclide_index(g, energy, nuclide, count, k_out, stream))


def xs_get_table(g, table, offset, count, host_dst):
    _check(lib.xs_get_table(g, table, offset, count, host_dst))


def xs_set_param(g, name: str, value: int):
    _check(lib.xs_set_param(g, name.encode(), value))


def xs_last_error() -> str:
    return lib.xs_last_error().decode(errors="replace")


def xs_hash_finalize(s: int) -> int:
    return lib.xs_hash_finalize(s)


def xs_free_grid(g):
    lib.xs_free_grid(g)


def xs_timing_enable(g, enable: bool):
    _check(lib.xs_timing_enable(g, int(enable)))


def xs_timing_read(g) -> xs_timing:
    t = xs_timing()
    _check(lib.xs_timing_read(g, C.byref(t)))
    return t


# --------------------------------------------------------------- presets
from .xs_presets import CONC_SEED, GRID_SEED, LOOKUP_SEED, PRESETS  # noqa: E402


def make_spec(n_isotopes, n_gridpoints, grid_type="unionized", hash_bins=0, material_rule=0,
              grid_seed=GRID_SEED, conc_seed=CONC_SEED, lookup_seed=LOOKUP_SEED,
              index_layout="auto", **_):
    gt = GRID_TYPES[grid_type] if isinstance(grid_type, str) else int(grid_type)
    il = INDEX_LAYOUTS[index_layout] if isinstance(index_layout, str) else int(index_layout)
    return xs_grid_spec(XS_ABI_VERSION, n_isotopes, n_gridpoints, gt,
                        hash_bins if gt == XS_GRID_HASH else 0, grid_seed, conc_seed,
                        lookup_seed, material_rule, il)


class Grid:
    """One replica of the XS tables on one CUDA device (torch-managed I/O)."""

    def __init__(self, handle: int, device: int):
        import torch
        self._h = handle
        self.device = torch.device("cuda", device)
        self.info = xs_grid_get_info(handle)
        self._ws = None

    @classmethod
    def from_spec(cls, device: int = 0, **spec_kw):
        import torch
        with torch.cuda.device(device):
            st = torch.cuda.current_stream().cuda_stream
            return cls(xs_init_grid(make_spec(**spec_kw), device, st), device)

    @classmethod
    def from_preset(cls, name: str, device: int = 0, **over):
        kw = dict(PRESETS[name])
        kw.update(over)
        return cls.from_spec(device=device, **kw)

    @classmethod
    def from_arrays(cls, grid, num_nucs, mats, concs, grid_type="unionized", hash_bins=0,
                    lookup_seed=LOOKUP_SEED, device: int = 0, index_layout="auto"):
        import numpy as np
        import torch
        grid = np.ascontiguousarray(grid, np.float64)
        num_nucs = np.ascontiguousarray(num_nucs, np.int32)
        mats = np.ascontiguousarray(mats, np.int32)
        concs = np.ascontiguousarray(concs, np.float64)
        I, N, six = grid.shape
        assert six == 6
        gt = GRID_TYPES[grid_type] if isinstance(grid_type, str) else int(grid_type)
        d = xs_grid_data(XS_ABI_VERSION, I, N, grid.ctypes.data, mats.shape[0], mats.shape[1],
                         num_nucs.ctypes.data, mats.ctypes.data, concs.ctypes.data, gt,
                         hash_bins, lookup_seed,
                         INDEX_LAYOUTS[index_layout] if isinstance(index_layout, str)
                         else int(index_layout), 0)
        with torch.cuda.device(device):
            st = torch.cuda.current_stream().cuda_stream
            return cls(xs_init_grid_data(d, device, st), device)

    def close(self):
        h, self._h = getattr(self, "_h", None), None
        if h:
            xs_free_grid(h)

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_param(self, name: str, value: int):
        xs_set_param(self._h, name, value)

    def timing(self, enable: bool = True):
        xs_timing_enable(self._h, enable)

    def timing_read(self) -> dict:
        t = xs_timing_read(self._h)
        return {k: getattr(t, k) for k, _ in xs_timing._fields_}

    def workspace_size(self, count: int, flags: int = 0) -> int:
        return xs_workspace_size(self._h, count, flags)

    def workspace(self, count: int, flags: int = 0):
        import torch
        n = xs_workspace_size(self._h, count, flags)
        if self._ws is None or self._ws.numel() < n:
            self._ws = torch.empty(max(n, 256), dtype=torch.uint8, device=self.device)
        return self._ws

    def _outputs(self, count, want, vsum, host=False):
        import torch
        dev = "cpu" if host else self.device
        pin = host and torch.cuda.is_available()
        res = {}

        def mk(name, shape, dt):
            if name in want:
                t = torch.empty(shape, dtype=dt, device=dev, pin_memory=pin)
                res[name] = t
                return t.data_ptr()
            return None
        o = xs_outputs(mk("macro_xs", (count, 5), torch.float64),
                       mk("energy", (count,), torch.float64), mk("mat", (count,), torch.int32),
                       mk("grid_index", (count,), torch.int64),
                       mk("verification", (count,), torch.int32), vsum.data_ptr())
        return o, res

    def _stream(self) -> int:
        """torch's current stream of the grid's device: workspace and outputs
        are allocated by torch's caching allocator, which orders their reuse
        on this stream, so every call is enqueued on it."""
        import torch
        return torch.cuda.current_stream(self.device).cuda_stream

    def lookup(self, first_id: int, count: int, sort: bool = False, baseline: bool = False,
               want=(), vsum=None, f32: bool = False):
        """A1-A8 for lookup ids [first_id, first_id+count) on the current stream
        (f32: the fp32 variant, XS_FLAG_F32).
        Returns (vsum tensor [2] uint64-as-int64 on device, dict of outputs)."""
        import torch
        flags = ((XS_FLAG_SORT if sort else 0) | (XS_FLAG_BASELINE if baseline else 0) |
                 (XS_FLAG_F32 if f32 else 0))
        if vsum is None:
            vsum = torch.zeros(2, dtype=torch.int64, device=self.device)
        o, res = self._outputs(count, want, vsum)
        ws = self.workspace(count, flags)
        xs_lookup_batch(self._h, first_id, count, flags, o, ws.data_ptr(), ws.numel(),
                        self._stream())
        return vsum, res

    def lookup_shard(self, first_id: int, count: int, shard: int, n_shards: int, want=(),
                     vsum=None, f32: bool = False, outputs=None):
        """Energy-range shard `shard` of `n_shards` of the sampled batch
        [first_id, first_id+count) (xs_lookup_batch_shard; A2 always on).
        Per-lookup outputs are batch-position indexed and written only for
        the shard's lookups; pass `outputs` (a dict from an earlier call) to
        let several shards fill the same tensors."""
        import torch
        flags = XS_FLAG_SORT | (XS_FLAG_F32 if f32 else 0)
        if vsum is None:
            vsum = torch.zeros(2, dtype=torch.int64, device=self.device)
        if outputs is None:
            o, res = self._outputs(count, want, vsum)
        else:
            res = outputs
            g = lambda k: res[k].data_ptr() if k in res else None  # noqa: E731
            o = xs_outputs(g("macro_xs"), g("energy"), g("mat"), g("grid_index"),
                           g("verification"), vsum.data_ptr())
        ws = self.workspace(count, flags)
        xs_lookup_batch_shard(self._h, first_id, count, shard, n_shards, flags, o,
                              ws.data_ptr(), ws.numel(), self._stream())
        return vsum, res

    def lookup_explicit(self, energy, mat, sort=False, want=(), vsum=None, f32: bool = False,
                        asynchronous: bool = False, workspace=None):
        """A2-A8 for caller-given (energy, material).  energy/mat are CUDA
        tensors (float64 / int32 or uint8 -> XS_FLAG_MAT_U8), or CPU tensors
        (then XS_FLAG_HOST_IO: staged copies inside the call, outputs returned
        on the host).  asynchronous=True (host tensors, pinned): XS_FLAG_HOST_ASYNC
        — the call returns before the work is done; synchronize the current
        stream before reading the outputs, and pass a different `workspace`
        (uint8 CUDA tensor of xs_workspace_size bytes) to consecutive calls
        so that the upload of one overlaps the lookups of the other."""
        import torch
        host = not energy.is_cuda
        if asynchronous and not host:
            raise ValueError("asynchronous=True takes host (pinned) tensors")
        io = (XS_FLAG_HOST_ASYNC if asynchronous else XS_FLAG_HOST_IO) if host else 0
        flags = ((XS_FLAG_SORT if sort else 0) | io | (XS_FLAG_F32 if f32 else 0) |
                 (XS_FLAG_MAT_U8 if mat.dtype == torch.uint8 else 0))
        count = energy.numel()
        if vsum is None:
            vsum = torch.zeros(2, dtype=torch.int64, device="cpu" if host else self.device)
        o, res = self._outputs(count, want, vsum, host=host)
        ws = workspace if workspace is not None else self.workspace(count, flags)
        xs_lookup_explicit(self._h, energy.data_ptr(), mat.data_ptr(), count, flags, o,
                           ws.data_ptr(), ws.numel(), self._stream())
        return vsum, res

    def lookup_history(self, first_particle: int, n_particles: int, lookups: int = 34,
                       sort: bool = False, want=(), vsum=None):
        """History mode (R19): n_particles x lookups chained lookups.
        Per-lookup outputs in `want` (macro_xs, energy, mat, verification) are
        [n_particles * lookups] (lookup i of particle q at q * lookups + i)."""
        import torch
        flags = XS_FLAG_SORT if sort else 0
        if vsum is None:
            vsum = torch.zeros(2, dtype=torch.int64, device=self.device)
        o, res = self._outputs(n_particles * lookups, want, vsum)
        n = xs_history_workspace_size(self._h, n_particles, flags)
        if self._ws is None or self._ws.numel() < n:
            self._ws = torch.empty(max(n, 256), dtype=torch.uint8, device=self.device)
        xs_lookup_history(self._h, first_particle, n_particles, lookups, flags, o,
                          self._ws.data_ptr(), self._ws.numel(), self._stream())
        return vsum, res

    def verify(self, macro_xs, vsum=None):
        import torch
        if vsum is None:
            vsum = torch.zeros(2, dtype=torch.int64, device=self.device)
        xs_verify(self._h, macro_xs.data_ptr(), macro_xs.shape[0], vsum.data_ptr(),
                  torch.cuda.current_stream(self.device).cuda_stream)
        return vsum

    def nuclide_index(self, energy, nuclide):
        import torch
        k = torch.empty(energy.numel(), dtype=torch.int32, device=self.device)
        xs_nuclide_index(self._h, energy.data_ptr(), nuclide.data_ptr(), energy.numel(),
                         k.data_ptr(), torch.cuda.current_stream(self.device).cuda_stream)
        return k

    def table(self, which: int, offset: int = 0, count: int | None = None):
        import numpy as np
        i = self.info
        lens = {XS_TABLE_NUCLIDE_GRID: i.n_isotopes * i.n_gridpoints * 6,
                XS_TABLE_UNION_ENERGY: i.n_union, XS_TABLE_INDEX_GRID: i.index_grid_len,
                XS_TABLE_NUM_NUCS: i.n_mats, XS_TABLE_MATS: i.n_mats * i.max_num_nucs,
                XS_TABLE_CONCS: i.n_mats * i.max_num_nucs,
                XS_TABLE_INDEX_GRID_T: i.index_grid_len if i.index_layout & 2 else 0,
                XS_TABLE_INTERVALS: i.n_isotopes * i.n_gridpoints * 14,
                XS_TABLE_INTERVALS32: i.n_isotopes * i.n_gridpoints * 10,
                XS_TABLE_INTERVALS_U: i.n_isotopes * i.n_gridpoints * 12}
        dt = np.int32 if which in (XS_TABLE_INDEX_GRID, XS_TABLE_NUM_NUCS, XS_TABLE_MATS,
                                   XS_TABLE_INDEX_GRID_T) \
            else np.float64
        if count is None:
            count = lens[which] - offset
        out = np.empty(count, dt)
        xs_get_table(self._h, which, offset, count, out.ctypes.data)
        return out


def hash_of(vsum) -> int:
    """A9 epilogue on a (globally reduced) vsum tensor/list: sum v mod 999983."""
    s = int(vsum[0])
    return xs_hash_finalize(s & 0xFFFFFFFFFFFFFFFF)
