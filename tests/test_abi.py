"""CPU-side checks of the C-ABI library (no compute calls: there is no GPU here)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "bzk.h")


def declared_symbols():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(bzk_[a-z0-9_]+)\s*\(", src)))


@pytest.fixture(scope="module")
def libbzk():
    from paper_conf_asplos_lucw0cz25_b200 import build
    build.build()
    from paper_conf_asplos_lucw0cz25_b200 import bzk
    return bzk.lib()


def test_header_declares_the_boundary():
    syms = declared_symbols()
    for s in ("bzk_create", "bzk_destroy", "bzk_prove", "bzk_prove_ragged", "bzk_sync", "bzk_workspace_size",
              "bzk_strerror", "bzk_last_error"):
        assert s in syms


def test_library_exports_every_declared_symbol(libbzk):
    for s in declared_symbols():
        assert hasattr(libbzk, s), s
    from paper_conf_asplos_lucw0cz25_b200 import bzk
    assert sorted(bzk.EXPORTS) == declared_symbols()


def test_library_is_sm100a(libbzk):
    import subprocess
    from paper_conf_asplos_lucw0cz25_b200 import bzk
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", bzk.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


def test_version_and_strerror(libbzk):
    from paper_conf_asplos_lucw0cz25_b200 import bzk
    assert "sm_100a" in bzk.bzk_version()
    assert libbzk.bzk_strerror(bzk.BZK_ENONCANON).decode() == "non-canonical input element"


def test_argument_errors_without_gpu(libbzk):
    from paper_conf_asplos_lucw0cz25_b200 import bzk
    # null destinations are rejected before any launch
    assert libbzk.bzk_generate(None, 1, 2, 3, 0, 0, 0, None) == bzk.BZK_EINVAL
    assert libbzk.bzk_debug_field(9, 1, None, None, None, None) == bzk.BZK_EINVAL
    h = ctypes.c_void_p()
    assert libbzk.bzk_create(0, 0, None) == bzk.BZK_EINVAL
    # no GPU in this container: creation fails cleanly instead of crashing
    st = libbzk.bzk_create(0, 0, ctypes.byref(h))
    assert st in (bzk.BZK_OK, bzk.BZK_ECUDA)
    if st == bzk.BZK_OK:
        libbzk.bzk_destroy(h)


def test_module_entry_points_reject_bad_arguments_without_gpu(libbzk):
    """NEXT-3 / NEXT-4 entry points: NULL context / destination are rejected before any CUDA call."""
    from paper_conf_asplos_lucw0cz25_b200 import bzk
    b = bzk.bzk_merkle_batch(4, 0, 0, 0, 1, None, 0, 0, None, None)
    assert libbzk.bzk_merkle(None, ctypes.byref(b), None) == bzk.BZK_EINVAL
    assert libbzk.bzk_generate_blocks(None, 1, 4, 0, 0, None) == bzk.BZK_EINVAL
    h = ctypes.c_void_p()
    assert libbzk.bzk_encoder_create(None, None, ctypes.byref(h)) == bzk.BZK_EINVAL
    assert libbzk.bzk_encode(None, None, None, 1, 0, 0, None) == bzk.BZK_EINVAL
    libbzk.bzk_encoder_destroy(None)   # no-op
    c = bzk.bzk_commit(4, 0, None, None, None, None)
    sb = bzk.bzk_batch()
    assert libbzk.bzk_commit_prove(None, None, ctypes.byref(c), ctypes.byref(sb), None) == bzk.BZK_EINVAL
    assert libbzk.bzk_debug_gl(0, 1, None, None, None, None) == bzk.BZK_EINVAL


def test_abi_struct_layouts_match_header():
    """ctypes mirrors of the ABI structs have the sizes the C compiler gives the header's structs."""
    import subprocess
    import tempfile
    from paper_conf_asplos_lucw0cz25_b200 import bzk
    src = """#include <stdio.h>
#include "bzk.h"
int main(void) { printf("%zu %zu %zu %zu %zu\\n", sizeof(bzk_batch), sizeof(bzk_merkle_batch), sizeof(bzk_csr),
                        sizeof(bzk_code), sizeof(bzk_commit)); return 0; }
"""
    with tempfile.TemporaryDirectory() as d:
        c = os.path.join(d, "s.c")
        open(c, "w").write(src)
        exe = os.path.join(d, "s")
        subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), c, "-o", exe])
        sizes = [int(x) for x in subprocess.check_output([exe]).split()]
    assert sizes == [ctypes.sizeof(bzk.bzk_batch), ctypes.sizeof(bzk.bzk_merkle_batch), ctypes.sizeof(bzk.bzk_csr),
                     ctypes.sizeof(bzk.bzk_code), ctypes.sizeof(bzk.bzk_commit)]


def test_product_package_does_not_touch_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_asplos_lucw0cz25_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
                assert "oracle.c" not in txt and "liboracle" not in txt, f
