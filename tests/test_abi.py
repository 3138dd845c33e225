"""CPU checks of the boundary: libxs.so builds for sm_100a, loads, exports
every symbol include/xs.h declares, and fails loudly (no CPU fallback) when
there is no GPU.  No compute calls are made here."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    with open(os.path.join(ROOT, "include", "xs.h")) as f:
        src = f.read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:const\s+)?\w+\*?\s+\*?(xs_\w+)\s*\(", src, flags=re.M)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_sc_tianscd23_b200 import build
    path = build.build()
    return ctypes.CDLL(path)


def test_header_declares_the_entry_points():
    names = _declared()
    for n in ("xs_init_grid", "xs_lookup_batch", "xs_verify", "xs_lookup_explicit",
              "xs_workspace_size", "xs_free_grid", "xs_last_error", "xs_hash_finalize"):
        assert n in names, n


def test_library_exports_every_declared_symbol(lib):
    for n in _declared():
        assert hasattr(lib, n), f"libxs.so does not export {n}"
    out = subprocess.run(["nm", "-D", "--defined-only", os.path.join(
        ROOT, "paper_conf_sc_tianscd23_b200", "libxs.so")], capture_output=True, text=True).stdout
    for n in _declared():
        assert re.search(rf"\bT {n}$", out, flags=re.M), n


def test_library_is_sm100a(lib):
    so = os.path.join(ROOT, "paper_conf_sc_tianscd23_b200", "libxs.so")
    out = subprocess.run(["cuobjdump", "--list-elf", so], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_python_binding_names_match_header():
    import paper_conf_sc_tianscd23_b200.xs as X
    assert X.xs_abi_version() == 1
    for n in _declared():
        assert hasattr(X, n), f"binding lacks {n}"
    assert X.xs_hash_finalize(50951281) == 952131


def test_no_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    import paper_conf_sc_tianscd23_b200.xs as X
    with pytest.raises(X.XSError) as e:
        X.xs_init_grid(X.make_spec(12, 1000, material_rule=1), 0, 0)
    assert e.value.status in (3, 4)  # XS_ERR_CUDA / XS_ERR_UNSUPPORTED, never a CPU result


def test_invalid_arguments_without_gpu():
    import paper_conf_sc_tianscd23_b200.xs as X
    with pytest.raises(X.XSError) as e:
        X.xs_init_grid(X.make_spec(100, 1000, material_rule=0), 0, 0)   # rule 0 needs 68/355
    assert e.value.status == 1
    with pytest.raises(X.XSError):
        X.xs_workspace_size(None, 10, 0)


def test_product_and_oracle_share_no_code():
    """oracle/ and the product path import / include nothing of each other;
    the only shared module is the input generator gen/."""
    pkg = os.path.join(ROOT, "paper_conf_sc_tianscd23_b200")
    for dirpath, _, files in os.walk(pkg):
        for fn in files:
            if fn.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                with open(os.path.join(dirpath, fn)) as f:
                    s = f.read()
                assert not re.search(r"^\s*(import|from)\s+oracle\b", s, flags=re.M), fn
                assert "xs_oracle" not in s and "rs_oracle" not in s, fn
    for fn in os.listdir(os.path.join(ROOT, "oracle")):
        if fn.endswith((".py", ".c", ".h")):
            with open(os.path.join(ROOT, "oracle", fn)) as f:
                s = f.read()
            assert not re.search(r"(import|from)\s+paper_conf_sc_tianscd23_b200", s), fn
            assert not re.search(r'#include\s+"[^"]*\b[xr]s\.h"', s), fn
            assert "libxs" not in s, fn


# ------------------------------------------------------------ RSBench (rs.h)
def _declared_rs():
    with open(os.path.join(ROOT, "include", "rs.h")) as f:
        src = f.read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:const\s+)?\w+\*?\s+\*?(rs_\w+)\s*\(", src, flags=re.M)))


def test_rs_header_and_exports(lib):
    names = _declared_rs()
    for n in ("rs_init", "rs_workspace_size", "rs_lookup_batch", "rs_free"):
        assert n in names, n
    out = subprocess.run(["nm", "-D", "--defined-only", os.path.join(
        ROOT, "paper_conf_sc_tianscd23_b200", "libxs.so")], capture_output=True, text=True).stdout
    import paper_conf_sc_tianscd23_b200.rs as R
    for n in names:
        assert re.search(rf"\bT {n}$", out, flags=re.M), n
        assert hasattr(R, n), f"binding lacks {n}"


def test_rs_fails_loudly_without_gpu():
    import torch
    import paper_conf_sc_tianscd23_b200.rs as R
    import paper_conf_sc_tianscd23_b200.xs as X
    with pytest.raises(X.XSError) as e:
        R.rs_init(R.make_spec(12, material_rule=1, numL=3), 0, 0)
    assert e.value.status == 4                        # numL != 4: unsupported
    if torch.cuda.is_available():
        return
    with pytest.raises(X.XSError) as e:
        R.rs_init(R.make_spec(12, material_rule=1), 0, 0)
    assert e.value.status in (3, 4)
