"""The C-ABI library builds for sm_100a, loads without a GPU, and exports every call include/sr.h declares."""
import ctypes
import os
import re

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "sr.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(sr_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_the_boundary_calls():
    names = _declared()
    for must in ("sr_create", "sr_infer", "sr_train_step", "sr_psnr_gain", "sr_infer_rows", "sr_publish",
                 "sr_pool_push", "sr_train_grad", "sr_train_apply", "sr_sample_batch"):
        assert must in names


def test_library_exports_every_declared_symbol():
    from paper_conf_sigcomm_kimjyyh20_b200 import build
    lib_path = build.build(force=False, verbose=False)
    lib = ctypes.CDLL(lib_path)
    missing = [n for n in _declared() if not hasattr(lib, n)]
    assert not missing, missing


def test_binding_covers_every_declared_symbol():
    from paper_conf_sigcomm_kimjyyh20_b200 import _lib
    missing = [n for n in _declared() if n not in _lib._SIGS]
    assert not missing, missing


def test_product_path_has_no_oracle_or_cpu_fallback():
    """Nothing under the package imports the oracle; loading fails loudly without the CUDA library."""
    pkg = os.path.join(ROOT, "paper_conf_sigcomm_kimjyyh20_b200")
    for dirpath, _, files in os.walk(pkg):
        for fn in files:
            if fn.endswith((".py", ".cu", ".cuh", ".h")):
                src = open(os.path.join(dirpath, fn)).read()
                for ln in src.splitlines():
                    if re.match(r"\s*(import|from)\s", ln) or ln.strip().startswith("#include"):
                        assert "oracle" not in ln, (fn, ln)
    from paper_conf_sigcomm_kimjyyh20_b200 import _lib
    try:
        _lib._lib = None
        _lib.load("/nonexistent/libsr.so")
        raise AssertionError("load() of a missing library must raise")
    except RuntimeError:
        pass
    finally:
        _lib._lib = None


def test_nccl_unique_id_and_missing_library():
    """sr_nccl_unique_id draws a 128-byte id through the dlopen'ed libnccl (no GPU needed), returns SR_E_INVAL for a
    short buffer, and SR_E_NCCL when libnccl cannot be loaded (SR_NCCL_LIB pointing nowhere, fresh process)."""
    import subprocess
    import sys
    code = ("import ctypes, sys; sys.path.insert(0, %r); from paper_conf_sigcomm_kimjyyh20_b200 import load; "
            "lib = load(); b = ctypes.create_string_buffer(128); s = ctypes.create_string_buffer(16); "
            "print(lib.sr_nccl_unique_id(b, 128), lib.sr_nccl_unique_id(s, 16), int(any(b.raw)))" % ROOT)
    ok = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=120)
    assert ok.stdout.split() == ["0", "-1", "1"], ok.stdout + ok.stderr
    env = dict(os.environ, SR_NCCL_LIB="/nonexistent/libnccl.so.2")
    bad = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=120, env=env)
    assert bad.stdout.split()[0] == "-4", bad.stdout + bad.stderr
