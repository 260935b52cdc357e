"""CPU-only checks of the C-ABI library: it loads, exports every symbol include/*.h
declares, and host-side argument validation works without a GPU."""
import ctypes
import glob
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    from paper_conf_hpdc_yudztt0c22_b200 import _build, szx
    _build.build()
    return szx.lib()


def _declared():
    names = set()
    for h in glob.glob(os.path.join(ROOT, "include", "*.h")):
        src = open(h).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        for m in re.finditer(r"\b(szx_[a-z0-9_]+)\s*\(", src):
            names.add(m.group(1))
    return names


def test_header_declarations_exported(L):
    from paper_conf_hpdc_yudztt0c22_b200 import szx
    decl = _declared()
    assert len(decl) >= 15
    out = subprocess.run(["nm", "-D", "--defined-only", szx.LIB_PATH], capture_output=True, text=True).stdout
    exported = {l.split()[-1] for l in out.splitlines() if l.strip()}
    missing = decl - exported
    assert not missing, missing
    assert set(szx.EXPORTED) == decl


def test_library_is_sm100a(L):
    from paper_conf_hpdc_yudztt0c22_b200 import szx
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", szx.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_bounds_and_validation_without_gpu(L):
    from paper_conf_hpdc_yudztt0c22_b200 import szx
    import oracle
    for n in (0, 1, 127, 128, 129, 10_000_019):
        for dt in (0, 1):
            assert szx.compress_bound(n, dt, 128) == oracle.compress_bound(n, dt, 128)
    # argument errors are reported before touching the device
    assert L.szx_compress(None, 0, 10, 0, -1.0, 128, None, 0, None) == -1
    assert L.szx_compress(None, 0, 10, 0, float("nan"), 128, None, 0, None) == -1
    assert L.szx_compress(None, 0, 10, 2, 1e-3, 128, None, 0, None) == -1
    assert L.szx_compress(None, 0, 10, 0, 1e-3, 100, None, 0, None) == -1
    assert L.szx_compress(None, 0, 10, 0, 1e-3, 128, ctypes.c_void_p(8), 0, None) == -1  # misaligned
    assert L.szx_compress_workspace_bytes(1000, 0, 100) == 0
    assert L.szx_strerror(-3) == b"corrupt stream"


def test_header_parse_matches_oracle_stream(L):
    import numpy as np
    import oracle
    from paper_conf_hpdc_yudztt0c22_b200 import szx
    x = np.linspace(-3, 7, 5000, dtype=np.float32)
    s = oracle.compress(x, 1e-3, oracle.REL, 128)
    h = szx.read_header(s.tobytes())
    ho = oracle.read_header(s)
    assert (h.n, h.block_size, h.n_nonconst, h.payload_bytes) == (ho["n"], ho["b"], ho["nnc"], ho["payload_bytes"])
    assert h.eb_abs == ho["eb_abs"] and h.stream_bytes == s.size
    bad = bytearray(s[:64].tobytes()); bad[0] = 0
    with pytest.raises(szx.SZxError):
        szx.read_header(bytes(bad))
