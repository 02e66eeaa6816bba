"""The C-ABI library loads and exports every symbol include/lcf.h declares; host
pure functions agree with the oracle and FORMAT.md (-m "not gpu": no compute
calls)."""
import ctypes
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    from paper_conf_asplos_azamifb25_b200 import build, lcf
    build.build()
    return lcf


def declared_functions():
    with open(os.path.join(ROOT, "include", "lcf.h")) as f:
        src = f.read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(lcf_[a-z_]+)\s*\(", src)))


def test_exports_every_declared_symbol(L):
    names = declared_functions()
    assert len(names) >= 10
    lib = ctypes.CDLL(L.LIB_PATH)
    for n in names:
        assert hasattr(lib, n), n


def test_library_is_sm100a(L):
    out = os.popen(f"cuobjdump --list-elf {L.LIB_PATH} 2>&1").read()
    assert "sm_100a" in out


@pytest.mark.parametrize("algo", ["SPspeed", "SPratio", "DPspeed", "DPratio"])
def test_max_size_and_chunk_count_match_oracle(L, orc, algo):
    for n in [0, 8, 16384, 16384 * 3 + 8, 25920000, 301989888, 1123815468 // 4 * 4]:
        if algo.startswith("DP") and n % 8:
            continue
        assert L.lcf_max_compressed_size(algo, None, n) == orc.max_compressed_size(algo, n)
        wb = 4 if algo.startswith("SP") else 8
        expect = 2 * -(-(n // wb) // 2048) if algo == "DPratio" else -(-n // 16384)
        assert L.lcf_num_chunks(algo, n) == expect


def test_config_chunk_counts(L):
    """SURVEY §8(a) config table."""
    assert L.lcf_num_chunks("SPspeed", 512 * 512 * 4) == 64
    assert L.lcf_num_chunks("SPspeed", 1800 * 3600 * 4) == 1583
    assert L.lcf_num_chunks("DPspeed", 256 * 384 * 384 * 8) == 18432
    assert L.lcf_num_chunks("DPratio", 256 * 384 * 384 * 8) == 36864
    assert L.lcf_num_chunks("SPspeed", 512 ** 3 * 4) == 32768
    assert L.lcf_num_chunks("SPspeed", 280953867 * 4) == 68593


def test_no_device_means_error_not_fallback(L):
    """Without a GPU the library refuses to compute (no CPU fallback)."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    x = np.zeros(1024, np.float32)
    out = np.zeros(1 << 16, np.uint8)
    with pytest.raises(L.LcfError) as e:
        L.lcf_compress_host("SPspeed", None, x, x.nbytes, out, out.nbytes, stream=0)
    assert e.value.status == 5


def test_cpu_library_exports_every_declared_symbol():
    """liblcf_cpu.so (include/lcf_cpu.h): separate from liblcf.so, which must not
    export any lcf_cpu_* symbol (the GPU library has no CPU codec path)."""
    from paper_conf_asplos_azamifb25_b200 import build
    build.build_cpu()
    with open(os.path.join(ROOT, "include", "lcf_cpu.h")) as f:
        src = re.sub(r"/\*.*?\*/", "", f.read(), flags=re.S)
    names = sorted(set(re.findall(r"\b(lcf_cpu_[a-z_]+)\s*\(", src)))
    assert len(names) == 3
    lib = ctypes.CDLL(build.CPU_LIB)
    for n in names:
        assert hasattr(lib, n), n
    gpu = ctypes.CDLL(build.LIB)
    for n in names:
        assert not hasattr(gpu, n), n


@pytest.mark.parametrize("algo", ["SPspeed", "SPratio", "DPspeed", "DPratio"])
def test_cpu_max_size_matches(L, algo):
    from paper_conf_asplos_azamifb25_b200 import lcf_cpu
    for n in [0, 8, 16384, 16384 * 3 + 8, 25920000, 301989888]:
        assert lcf_cpu.lcf_cpu_max_compressed_size(algo, n) == L.lcf_max_compressed_size(algo, None, n)
