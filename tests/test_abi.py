"""CPU-side checks of the boundary: libpfpl.so builds for sm_100a, loads
without a GPU and exports every function declared in include/pfpl.h; the
product path never touches oracle/ and fails loudly without CUDA."""
import ast
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_ipps_fallinadcb25_b200")


def _declared():
    src = open(os.path.join(ROOT, "include", "pfpl.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(pfpl_[a-z_0-9]+)\s*\(", src)))


@pytest.fixture(scope="module")
def libpath():
    from paper_conf_ipps_fallinadcb25_b200 import _build
    return _build.build()


def test_exports_every_declared_symbol(libpath):
    import ctypes
    L = ctypes.CDLL(libpath)
    names = _declared()
    assert len(names) >= 15
    for n in names:
        assert hasattr(L, n), n
    dyn = subprocess.run(["nm", "-D", "--defined-only", libpath], capture_output=True, text=True).stdout
    for n in names:
        assert re.search(rf"\bT {n}\b", dyn), n


def test_sm100a_code_only(libpath):
    out = subprocess.run(["cuobjdump", "--list-elf", libpath], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_host_only_calls_without_gpu(libpath):
    import ctypes
    import paper_conf_ipps_fallinadcb25_b200 as pk
    L = pk.lib()
    assert L.pfpl_max_compressed_bytes(4096, 0) == 48 + 4 + 16384
    assert L.pfpl_max_compressed_bytes(0, 1) == 48
    assert L.pfpl_strerror(-4) == b"corrupt stream"
    assert b"sm_100a" in L.pfpl_version()
    # header parsing (host-only)
    hdr = b"PFPL" + bytes([1, 0, 0, 0]) + (5).to_bytes(8, "little") + bytes(24) + \
        (16384).to_bytes(8, "little")
    info = pk.peek_header(hdr)
    assert info["n"] == 5 and info["dtype"] == 0
    with pytest.raises(pk.PFPLError):
        pk.peek_header(b"XXXX" + hdr[4:])


def test_product_fails_loudly_on_cpu_tensors():
    import torch
    import paper_conf_ipps_fallinadcb25_b200 as pk
    with pytest.raises(pk.PFPLError):
        pk.compress(torch.zeros(10), "abs", 1e-3)


def test_product_never_imports_oracle():
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith(".py"):
                tree = ast.parse(open(os.path.join(dirpath, f)).read())
                for node in ast.walk(tree):
                    if isinstance(node, ast.Import):
                        assert all(not a.name.startswith("oracle") for a in node.names), f
                    if isinstance(node, ast.ImportFrom):
                        assert not (node.module or "").startswith("oracle"), f
            if f.endswith((".cu", ".cuh", ".h", ".c")):
                assert "oracle" not in open(os.path.join(dirpath, f)).read().lower(), f


def test_batch_and_host_bindings_need_no_gpu_for_empty_and_reject_cuda_only_args():
    """Python-side argument handling of the NEXT-4 bindings (no compute call)."""
    import torch
    import paper_conf_ipps_fallinadcb25_b200 as pk
    assert pk.compress_batch([]) == []
    assert pk.decompress_batch([]) == []
    with pytest.raises(pk.PFPLError):
        pk.compress_host(torch.zeros(8, 2).t(), "abs", 1e-3)     # non-contiguous host tensor
    with pytest.raises(pk.PFPLError):
        pk.compress_batch([torch.zeros(8)], "abs", 1e-3)       # host tensor where CUDA is required


def test_cpu_codec_exports_every_declared_symbol():
    """libpfpl_cpu.so exports every function of include/pfpl_cpu.h."""
    import ctypes
    from paper_conf_ipps_fallinadcb25_b200 import _build
    path = _build.build_cpu()
    src = re.sub(r"/\*.*?\*/", "", open(os.path.join(ROOT, "include", "pfpl_cpu.h")).read(), flags=re.S)
    names = sorted(set(re.findall(r"\b(pfpl_cpu_[a-z_0-9]+)\s*\(", src)))
    assert len(names) == 4
    L = ctypes.CDLL(path)
    for n in names:
        assert hasattr(L, n), n
    assert L.pfpl_cpu_max_compressed_bytes(4096, 0) == 48 + 4 + 16384
