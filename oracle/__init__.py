"""CPU ORACLE for the XSBench event-based macroscopic XS lookup.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` leg may import this
package.  The product path (``paper_conf_sc_tianscd23_b200``) never imports
it and shares no code with it; the single shared module is the seeded input
generator ``gen/xs_gen.h`` (inputs only, none of the method's arithmetic).

This is a thin ctypes binding over ``oracle/xs_oracle.c`` (plain serial C,
fp64, ``-O2 -ffp-contract=off``); every step it exposes cites its reading in
DESIGN.md and is pinned by ``tests/test_oracle_*.py``.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_ROOT = os.path.dirname(_HERE)
LIB_PATH = os.path.join(_HERE, "liboracle.so")
_SOURCES = [os.path.join(_HERE, "xs_oracle.c"), os.path.join(_HERE, "xs_oracle.h"),
            os.path.join(_ROOT, "gen", "xs_gen.cpp"), os.path.join(_ROOT, "gen", "xs_gen.h"),
            os.path.join(_HERE, "rs_oracle.c"), os.path.join(_HERE, "rs_oracle.h"),
            os.path.join(_ROOT, "gen", "rs_gen.cpp"), os.path.join(_ROOT, "gen", "rs_gen.h")]

UNIONIZED, NUCLIDE, HASH = 0, 1, 2
F32 = 0x10   # OR into a mode: the fp32 variant (R18)
# run() modes whose M output is an error scale of the binary64 result instead
# of M: SCALE_A = sum_j |x_c conc_j|, SCALE_S = sum_j conc_j
# (|hi.c| + |f| (|hi.c| + |lo.c|)) (R18's a-priori scale)
SCALE_A, SCALE_S = 0x20, 0x40
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so (C oracle + the shared input generator)."""
    stale = force or not os.path.exists(LIB_PATH) or any(
        os.path.getmtime(s) > os.path.getmtime(LIB_PATH) for s in _SOURCES)
    if not stale:
        return LIB_PATH
    objs = [LIB_PATH + s for s in (".oracle.o", ".gen.o", ".rs_oracle.o", ".rs_gen.o")]
    flags = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC"]
    subprocess.check_call(["gcc", *flags, "-std=c11", "-c", _SOURCES[0], "-o", objs[0]])
    subprocess.check_call(["g++", *flags, "-std=c++17", "-c", _SOURCES[2], "-o", objs[1]])
    subprocess.check_call(["gcc", *flags, "-std=c11", "-c", _SOURCES[4], "-o", objs[2]])
    subprocess.check_call(["g++", *flags, "-std=c++17", "-c", _SOURCES[6], "-o", objs[3]])
    subprocess.check_call(["g++", "-shared", "-o", LIB_PATH + ".tmp", *objs, "-lpthread", "-lm"])
    os.replace(LIB_PATH + ".tmp", LIB_PATH)
    for f in objs:
        os.remove(f)
    return LIB_PATH


def lib() -> C.CDLL:
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = C.CDLL(LIB_PATH)
            u64, i64, i32, d = C.c_uint64, C.c_int64, C.c_int32, C.c_double
            P = C.c_void_p
            sig = {
                "oracle_lcg_step": (u64, [u64]),
                "oracle_lcg_to_double": (d, [u64]),
                "oracle_fast_forward": (u64, [u64, u64]),
                "oracle_thresholds": (None, [P]),
                "oracle_pick_mat": (i32, [d]),
                "oracle_sample": (None, [u64, u64, P, P]),
                "oracle_grid_search": (i64, [P, i64, i64, d]),
                "oracle_upper_bound": (i64, [P, i64, d]),
                "oracle_create_spec": (P, [i32, i64, u64, u64, i32, u64, i32, C.c_int, P]),
                "oracle_create_arrays": (P, [i32, i64, P, i32, i32, P, P, P, u64, i32, P]),
                "oracle_free": (None, [P]),
                "oracle_n_isotopes": (i32, [P]),
                "oracle_n_gridpoints": (i64, [P]),
                "oracle_n_mats": (i32, [P]),
                "oracle_max_num_nucs": (i32, [P]),
                "oracle_union_len": (i64, [P]),
                "oracle_grid": (P, [P]),
                "oracle_union": (P, [P]),
                "oracle_num_nucs": (P, [P]),
                "oracle_mats": (P, [P]),
                "oracle_concs": (P, [P]),
                "oracle_nuclide_bracket": (i64, [P, i32, d]),
                "oracle_union_index": (i64, [P, d]),
                "oracle_index_grid_entry": (i32, [P, i64, i32]),
                "oracle_index_grid_sweep": (C.c_int, [P, P]),
                "oracle_hash_bin": (i64, [P, d]),
                "oracle_hash_entry": (i32, [P, i64, i32]),
                "oracle_hash_bracket": (i64, [P, i64, i32, d]),
                "oracle_micro_xs": (None, [P, i32, i64, d, P]),
                "oracle_macro_xs": (None, [P, d, i32, C.c_int, P, P]),
                "oracle_verify": (C.c_int, [P]),
                "oracle_micro_xs_f32": (None, [P, i32, i64, d, P]),
                "oracle_macro_xs_f32": (None, [P, d, i32, C.c_int, P, P]),
                "oracle_lookup": (None, [P, u64, C.c_int, P, P, P, P, P]),
                "oracle_run": (u64, [P, u64, u64, C.c_int, C.c_int, P, P, P, P, P]),
                "oracle_run_explicit": (u64, [P, P, P, u64, C.c_int, C.c_int, P, P]),
                "oracle_run_history": (u64, [P, u64, u64, i32, C.c_int, C.c_int, P, P, P, P]),
                "oracle_hash_finalize": (u64, [u64]),
                "oracle_macro_scales": (None, [P, d, i32, P, P]),
                "oracle_index_grid_rows": (None, [P, i64, i64, P]),
                "oracle_hash_grid": (None, [P, P]),
                "xsgen_num_nucs": (C.c_int, [i32, i32, P]),
                "xsgen_max_num_nucs": (i32, [i32, i32]),
                "xsgen_mats": (C.c_int, [i32, i32, i32, P]),
                "xsgen_concs": (C.c_int, [u64, P, i32, P]),
                "xsgen_nuclide_grid": (C.c_int, [i32, i64, u64, P, C.c_int]),
                # RSBench oracle (rs_oracle.h, R20-R27)
                "rs_oracle_fast_exp": (d, [d]),
                "rs_oracle_fast_cexp": (None, [d, d, P, P]),
                "rs_oracle_faddeeva": (None, [d, d, P, P]),
                "rs_oracle_sigT_factors": (None, [P, d, P, P]),
                "rs_oracle_abrarov": (None, [d, d, d, d, P, P]),
                "rs_oracle_asymptotic": (None, [d, d, P, P]),
                "rs_oracle_abrarov_constants": (None, [P, P, P, P]),
                "rs_oracle_create": (P, [i32, i32, i32, i32, i32, u64, u64, i32, P]),
                "rs_oracle_free": (None, [P]),
                "rs_oracle_n_nuclides": (i32, [P]),
                "rs_oracle_max_num_nucs": (i32, [P]),
                "rs_oracle_max_poles": (i32, [P]),
                "rs_oracle_max_windows": (i32, [P]),
                "rs_oracle_num_nucs": (P, [P]),
                "rs_oracle_mats": (P, [P]),
                "rs_oracle_concs": (P, [P]),
                "rs_oracle_n_poles": (P, [P]),
                "rs_oracle_n_windows": (P, [P]),
                "rs_oracle_poles": (P, [P]),
                "rs_oracle_l_value": (P, [P]),
                "rs_oracle_windows": (P, [P]),
                "rs_oracle_wrange": (P, [P]),
                "rs_oracle_k0rs": (P, [P]),
                "rs_oracle_window": (i32, [P, i32, d]),
                "rs_oracle_micro_xs": (None, [P, i32, d, P]),
                "rs_oracle_macro_xs": (None, [P, d, i32, P]),
                "rs_oracle_verify": (C.c_int, [P]),
                "rs_oracle_lookup": (None, [P, u64, P, P, P, P]),
                "rs_oracle_run": (u64, [P, u64, u64, C.c_int, P, P, P, P]),
            }
            for name, (res, args) in sig.items():
                f = getattr(L, name)
                f.restype = res
                f.argtypes = args
            _lib = L
    return _lib


def _ptr(a: np.ndarray | None):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


# ------------------------------------------------------------- free helpers
def lcg_step(s: int) -> int:
    return lib().oracle_lcg_step(s)


def lcg_to_double(s: int) -> float:
    return lib().oracle_lcg_to_double(s)


def fast_forward(s: int, n: int) -> int:
    return lib().oracle_fast_forward(s, n)


def thresholds() -> np.ndarray:
    T = np.zeros(12, np.float64)
    lib().oracle_thresholds(_ptr(T))
    return T


def pick_mat(roll: float) -> int:
    return lib().oracle_pick_mat(roll)


def sample(lookup_seed: int, i: int) -> tuple[float, int]:
    p, m = C.c_double(), C.c_int32()
    lib().oracle_sample(lookup_seed, i, C.byref(p), C.byref(m))
    return p.value, m.value


def grid_search(A: np.ndarray, lo: int, hi: int, q: float) -> int:
    A = np.ascontiguousarray(A, np.float64)
    return lib().oracle_grid_search(_ptr(A), lo, hi, q)


def upper_bound(A: np.ndarray, q: float) -> int:
    A = np.ascontiguousarray(A, np.float64)
    return lib().oracle_upper_bound(_ptr(A), len(A), q)


def verify(M) -> int:
    M = np.ascontiguousarray(M, np.float64)
    return lib().oracle_verify(_ptr(M))


def hash_finalize(S: int) -> int:
    return lib().oracle_hash_finalize(S)


# ------------------------------------------------------------- generator view
def gen_num_nucs(I: int, rule: int) -> np.ndarray:
    out = np.zeros(12, np.int32)
    if lib().xsgen_num_nucs(I, rule, _ptr(out)):
        raise ValueError("bad (I, rule)")
    return out


# ------------------------------------------------------------------ context
class Oracle:
    """An oracle context: problem data + the oracle's own U / HG tables."""

    def __init__(self, handle):
        self._h = handle
        L = lib()
        self.I = L.oracle_n_isotopes(handle)
        self.N = L.oracle_n_gridpoints(handle)
        self.n_mats = L.oracle_n_mats(handle)
        self.max_num_nucs = L.oracle_max_num_nucs(handle)
        self.NU = L.oracle_union_len(handle)

    @classmethod
    def from_spec(cls, n_isotopes, n_gridpoints, grid_seed=42, conc_seed=0, material_rule=0,
                  lookup_seed=1070, hash_bins=0, nthreads=0):
        err = C.c_int(0)
        h = lib().oracle_create_spec(n_isotopes, n_gridpoints, grid_seed, conc_seed,
                                     material_rule, lookup_seed, hash_bins, nthreads,
                                     C.byref(err))
        if not h:
            raise ValueError(f"oracle_create_spec failed (err {err.value})")
        return cls(h)

    @classmethod
    def from_arrays(cls, grid, num_nucs, mats, concs, lookup_seed=1070, hash_bins=0):
        grid = np.ascontiguousarray(grid, np.float64)
        I, N, six = grid.shape
        assert six == 6
        num_nucs = np.ascontiguousarray(num_nucs, np.int32)
        mats = np.ascontiguousarray(mats, np.int32)
        concs = np.ascontiguousarray(concs, np.float64)
        n_mats, mx = mats.shape
        err = C.c_int(0)
        h = lib().oracle_create_arrays(I, N, _ptr(grid), n_mats, mx, _ptr(num_nucs), _ptr(mats),
                                       _ptr(concs), lookup_seed, hash_bins, C.byref(err))
        if not h:
            raise ValueError(f"oracle_create_arrays failed (err {err.value})")
        return cls(h)

    def __del__(self):
        h, self._h = getattr(self, "_h", None), None
        if h and lib is not None:
            try:
                lib().oracle_free(h)
            except Exception:
                pass

    # views (copies) of the tables
    def grid(self) -> np.ndarray:
        a = np.ctypeslib.as_array(C.cast(lib().oracle_grid(self._h), C.POINTER(C.c_double)),
                                  shape=(self.I * self.N * 6,))
        return a.reshape(self.I, self.N, 6).copy()

    def union(self) -> np.ndarray:
        a = np.ctypeslib.as_array(C.cast(lib().oracle_union(self._h), C.POINTER(C.c_double)),
                                  shape=(self.NU,))
        return a.copy()

    def num_nucs(self) -> np.ndarray:
        return np.ctypeslib.as_array(C.cast(lib().oracle_num_nucs(self._h), C.POINTER(C.c_int32)),
                                     shape=(self.n_mats,)).copy()

    def mats(self) -> np.ndarray:
        return np.ctypeslib.as_array(C.cast(lib().oracle_mats(self._h), C.POINTER(C.c_int32)),
                                     shape=(self.n_mats, self.max_num_nucs)).copy()

    def concs(self) -> np.ndarray:
        return np.ctypeslib.as_array(C.cast(lib().oracle_concs(self._h), C.POINTER(C.c_double)),
                                     shape=(self.n_mats, self.max_num_nucs)).copy()

    # steps
    def nuclide_bracket(self, n: int, p: float) -> int:
        return lib().oracle_nuclide_bracket(self._h, n, p)

    def union_index(self, p: float) -> int:
        return lib().oracle_union_index(self._h, p)

    def index_grid_entry(self, e: int, n: int) -> int:
        return lib().oracle_index_grid_entry(self._h, e, n)

    def index_grid_sweep(self) -> np.ndarray:
        out = np.empty((self.NU, self.I), np.int32)
        if lib().oracle_index_grid_sweep(self._h, _ptr(out)):
            raise MemoryError
        return out

    def index_grid_rows(self, e0: int, e1: int) -> np.ndarray:
        """IG rows [e0, e1) by the definition (R6)."""
        out = np.empty((e1 - e0, self.I), np.int32)
        lib().oracle_index_grid_rows(self._h, e0, e1, _ptr(out))
        return out

    def hash_grid(self, B: int) -> np.ndarray:
        """The whole hash grid HG [B][I] (R7); B = the context's hash_bins."""
        out = np.empty((B, self.I), np.int32)
        lib().oracle_hash_grid(self._h, _ptr(out))
        return out

    def macro_scales(self, p: float, mat: int):
        """(A, S): Q12's sum_j |x_c conc_j| and R18's a-priori scale."""
        A = np.zeros(5, np.float64)
        S = np.zeros(5, np.float64)
        lib().oracle_macro_scales(self._h, p, mat, _ptr(A), _ptr(S))
        return A, S

    def hash_bin(self, p: float) -> int:
        return lib().oracle_hash_bin(self._h, p)

    def hash_entry(self, b: int, n: int) -> int:
        return lib().oracle_hash_entry(self._h, b, n)

    def hash_bracket(self, b: int, n: int, p: float) -> int:
        return lib().oracle_hash_bracket(self._h, b, n, p)

    def micro_xs(self, n: int, k: int, p: float) -> np.ndarray:
        xs = np.zeros(5, np.float64)
        lib().oracle_micro_xs(self._h, n, k, p, _ptr(xs))
        return xs

    def micro_xs_f32(self, n: int, k: int, p: float) -> np.ndarray:
        xs = np.zeros(5, np.float32)
        lib().oracle_micro_xs_f32(self._h, n, k, p, _ptr(xs))
        return xs

    def macro_xs(self, p: float, mat: int, mode: int = UNIONIZED):
        """mode may include F32 (the fp32 variant; M is the binary32 result widened)."""
        M = np.zeros(5, np.float64)
        gi = C.c_int64(0)
        if mode & F32:
            lib().oracle_macro_xs_f32(self._h, p, mat, mode & 0xF, _ptr(M), C.byref(gi))
        else:
            lib().oracle_macro_xs(self._h, p, mat, mode, _ptr(M), C.byref(gi))
        return M, gi.value

    def lookup(self, i: int, mode: int = UNIONIZED):
        p, m, gi, v = C.c_double(), C.c_int32(), C.c_int64(), C.c_int32()
        M = np.zeros(5, np.float64)
        lib().oracle_lookup(self._h, i, mode, C.byref(p), C.byref(m), C.byref(gi), _ptr(M),
                            C.byref(v))
        return dict(p=p.value, mat=m.value, grid_index=gi.value, M=M, v=v.value)

    def run(self, first: int, count: int, mode: int = UNIONIZED, nthreads: int = 1,
            outputs: bool = False):
        """Lookups [first, first+count).  Returns S (= sum v) or (S, dict of arrays)."""
        if not outputs:
            return lib().oracle_run(self._h, first, count, mode, nthreads, None, None, None,
                                    None, None)
        p = np.empty(count, np.float64)
        mat = np.empty(count, np.int32)
        gi = np.empty(count, np.int64)
        M = np.empty((count, 5), np.float64)
        v = np.empty(count, np.int32)
        S = lib().oracle_run(self._h, first, count, mode, nthreads, _ptr(p), _ptr(mat), _ptr(gi),
                             _ptr(M), _ptr(v))
        return S, dict(p=p, mat=mat, grid_index=gi, M=M, v=v)

    def run_history(self, first_particle: int, n_particles: int, lookups: int,
                    mode: int = UNIONIZED, nthreads: int = 1, outputs: bool = False):
        """History mode (R19): particles [first, first+n), `lookups`
        chained lookups each.  Returns S or (S, dict of [n*lookups] arrays)."""
        if not outputs:
            return lib().oracle_run_history(self._h, first_particle, n_particles, lookups, mode,
                                            nthreads, None, None, None, None)
        n = n_particles * lookups
        p = np.empty(n, np.float64)
        mat = np.empty(n, np.int32)
        M = np.empty((n, 5), np.float64)
        v = np.empty(n, np.int32)
        S = lib().oracle_run_history(self._h, first_particle, n_particles, lookups, mode,
                                     nthreads, _ptr(p), _ptr(mat), _ptr(M), _ptr(v))
        return S, dict(p=p, mat=mat, M=M, v=v)

    def run_explicit(self, p: np.ndarray, mat: np.ndarray, mode: int = UNIONIZED,
                     nthreads: int = 1, outputs: bool = True):
        """Caller-given lookups.  Returns (S, M, v), or S alone (outputs=False)."""
        p = np.ascontiguousarray(p, np.float64)
        mat = np.ascontiguousarray(mat, np.int32)
        if not outputs:
            return lib().oracle_run_explicit(self._h, _ptr(p), _ptr(mat), len(p), mode, nthreads,
                                             None, None)
        M = np.empty((len(p), 5), np.float64)
        v = np.empty(len(p), np.int32)
        S = lib().oracle_run_explicit(self._h, _ptr(p), _ptr(mat), len(p), mode, nthreads,
                                      _ptr(M), _ptr(v))
        return S, M, v


# ------------------------------------------------------------ RSBench oracle
def rs_fast_exp(x: float) -> float:
    return lib().rs_oracle_fast_exp(x)


def rs_fast_cexp(z: complex) -> complex:
    r, i = C.c_double(), C.c_double()
    lib().rs_oracle_fast_cexp(z.real, z.imag, C.byref(r), C.byref(i))
    return complex(r.value, i.value)


def rs_faddeeva(z: complex) -> complex:
    """RSBench's fast_nuclear_W(z) (R24)."""
    r, i = C.c_double(), C.c_double()
    lib().rs_oracle_faddeeva(z.real, z.imag, C.byref(r), C.byref(i))
    return complex(r.value, i.value)


def rs_abrarov(z: complex, e: complex) -> complex:
    """The |z| < 6 branch of fast_nuclear_W with e = e^{12 i z} supplied (R24)."""
    r, i = C.c_double(), C.c_double()
    lib().rs_oracle_abrarov(z.real, z.imag, e.real, e.imag, C.byref(r), C.byref(i))
    return complex(r.value, i.value)


def rs_abrarov_constants():
    """(a_n, (-1)^n, (n pi)^2, tau^2/sqrt(pi)) as the oracle holds them."""
    an, sg, dl = (np.zeros(10, np.float64) for _ in range(3))
    pf = C.c_double()
    lib().rs_oracle_abrarov_constants(_ptr(an), _ptr(sg), _ptr(dl), C.byref(pf))
    return an, sg, dl, pf.value


def rs_asymptotic(z: complex) -> complex:
    """The |z| >= 6 branch of fast_nuclear_W (R24)."""
    r, i = C.c_double(), C.c_double()
    lib().rs_oracle_asymptotic(z.real, z.imag, C.byref(r), C.byref(i))
    return complex(r.value, i.value)


def rs_sigT_factors(k0, E: float) -> np.ndarray:
    """The four phase factors (cos 2phi_l, -sin 2phi_l) as complex (R23)."""
    k0 = np.ascontiguousarray(k0, np.float64)
    fr = np.zeros(4, np.float64)
    fi = np.zeros(4, np.float64)
    lib().rs_oracle_sigT_factors(_ptr(k0), E, _ptr(fr), _ptr(fi))
    return fr + 1j * fi


class RSOracle:
    """RSBench problem data (gen/rs_gen.h) + the serial multipole lookup
    (oracle/rs_oracle.c, R20-R27)."""

    def __init__(self, n_nuclides=355, avg_n_poles=1000, avg_n_windows=100, numL=4,
                 material_rule=0, seed=42, lookup_seed=1070, doppler=1):
        err = C.c_int(0)
        self._h = lib().rs_oracle_create(n_nuclides, avg_n_poles, avg_n_windows, numL,
                                         material_rule, seed, lookup_seed, doppler, C.byref(err))
        if not self._h:
            raise ValueError(f"rs_oracle_create failed (err {err.value})")
        L = lib()
        self.I = n_nuclides
        self.numL = numL
        self.doppler = doppler
        self.max_num_nucs = L.rs_oracle_max_num_nucs(self._h)
        self.P = L.rs_oracle_max_poles(self._h)
        self.W = L.rs_oracle_max_windows(self._h)

    def __del__(self):
        h, self._h = getattr(self, "_h", None), None
        if h and lib is not None:
            try:
                lib().rs_oracle_free(h)
            except Exception:
                pass

    def _view(self, fn, ctype, shape):
        a = np.ctypeslib.as_array(C.cast(getattr(lib(), fn)(self._h), C.POINTER(ctype)),
                                  shape=(int(np.prod(shape)),))
        return a.reshape(shape)

    # copies of the inputs; the writable views let pins edit the data in place
    def num_nucs(self):
        return self._view("rs_oracle_num_nucs", C.c_int32, (12,)).copy()

    def mats(self):
        return self._view("rs_oracle_mats", C.c_int32, (12, self.max_num_nucs)).copy()

    def concs(self):
        return self._view("rs_oracle_concs", C.c_double, (12, self.max_num_nucs)).copy()

    def n_poles(self):
        return self._view("rs_oracle_n_poles", C.c_int32, (self.I,)).copy()

    def n_windows(self):
        return self._view("rs_oracle_n_windows", C.c_int32, (self.I,)).copy()

    def poles(self, writable=False):
        v = self._view("rs_oracle_poles", C.c_double, (self.I, self.P, 8))
        return v if writable else v.copy()

    def l_value(self, writable=False):
        v = self._view("rs_oracle_l_value", C.c_int32, (self.I, self.P))
        return v if writable else v.copy()

    def windows(self, writable=False):
        v = self._view("rs_oracle_windows", C.c_double, (self.I, self.W, 3))
        return v if writable else v.copy()

    def wrange(self, writable=False):
        v = self._view("rs_oracle_wrange", C.c_int32, (self.I, self.W, 2))
        return v if writable else v.copy()

    def k0rs(self, writable=False):
        v = self._view("rs_oracle_k0rs", C.c_double, (self.I, self.numL))
        return v if writable else v.copy()

    # steps
    def window(self, nuc: int, E: float) -> int:
        return lib().rs_oracle_window(self._h, nuc, E)

    def micro_xs(self, nuc: int, E: float) -> np.ndarray:
        m = np.zeros(4, np.float64)
        lib().rs_oracle_micro_xs(self._h, nuc, E, _ptr(m))
        return m

    def macro_xs(self, E: float, mat: int) -> np.ndarray:
        M = np.zeros(4, np.float64)
        lib().rs_oracle_macro_xs(self._h, E, mat, _ptr(M))
        return M

    @staticmethod
    def verify(M) -> int:
        M = np.ascontiguousarray(M, np.float64)
        return lib().rs_oracle_verify(_ptr(M))

    def lookup(self, i: int):
        E, m, v = C.c_double(), C.c_int32(), C.c_int32()
        M = np.zeros(4, np.float64)
        lib().rs_oracle_lookup(self._h, i, C.byref(E), C.byref(m), _ptr(M), C.byref(v))
        return dict(E=E.value, mat=m.value, M=M, v=v.value)

    def run(self, first: int, count: int, nthreads: int = 1, outputs: bool = False):
        """Lookups [first, first+count).  Returns S (= sum v) or (S, dict)."""
        if not outputs:
            return lib().rs_oracle_run(self._h, first, count, nthreads, None, None, None, None)
        E = np.empty(count, np.float64)
        mat = np.empty(count, np.int32)
        M = np.empty((count, 4), np.float64)
        v = np.empty(count, np.int32)
        S = lib().rs_oracle_run(self._h, first, count, nthreads, _ptr(E), _ptr(mat), _ptr(M),
                                _ptr(v))
        return S, dict(E=E, mat=mat, M=M, v=v)
