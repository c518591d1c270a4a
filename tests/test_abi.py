"""The C-ABI library loads on CPU and exports every symbol include/seastar.h declares (no compute)."""
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    src = open(os.path.join(ROOT, "include", "seastar.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*(?:const\s+)?[A-Za-z_][A-Za-z0-9_]*\**\s+\**(seastar_[a-z0-9_]+)\s*\(", src, flags=re.M)
    return sorted(set(names))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_eurosys_wumcjlzcy21_b200 import build as B
    B.build()
    from paper_conf_eurosys_wumcjlzcy21_b200 import _lib
    return _lib


def test_header_parsed():
    names = declared_functions()
    assert "seastar_graph_create" in names and "seastar_gat_bwd" in names and len(names) >= 30


def test_every_declared_symbol_is_exported_and_bound(lib):
    so = lib.load()
    for name in declared_functions():
        assert hasattr(so, name), f"libseastar.so does not export {name}"
        assert name in lib.exported_symbols(), f"_lib.py has no binding for {name}"


def test_abi_version_and_no_cpu_fallback(lib):
    assert lib.seastar_abi_version() == 2
    import torch
    if not torch.cuda.is_available():
        # without a GPU every compute entry must fail loudly, never fall back to the CPU
        with pytest.raises(lib.SeastarError):
            lib.seastar_device_check()


def test_sm100a_cubin_only(lib):
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", lib.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out and "sm_90" not in out
