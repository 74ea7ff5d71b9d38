import ctypes
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (run with -m gpu under gpurun)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def hwcrc(tmp_path_factory):
    """The SSE4.2 crc32 instruction: an implementation independent of oracle/ and of the GPU path."""
    d = tmp_path_factory.mktemp("hwcrc")
    so = str(d / "hwcrc.so")
    subprocess.check_call(["gcc", "-O2", "-msse4.2", "-shared", "-fPIC", "-o", so,
                           os.path.join(ROOT, "tests", "helpers", "hwcrc.c")])
    lib = ctypes.CDLL(so)
    lib.hw_crc32c.restype = ctypes.c_uint32
    lib.hw_crc32c.argtypes = [ctypes.c_void_p, ctypes.c_size_t]

    def crc(data):
        import numpy as np
        a = np.ascontiguousarray(np.frombuffer(bytes(data), dtype=np.uint8) if not isinstance(data, np.ndarray)
                                 else data.view(np.uint8).reshape(-1))
        return int(lib.hw_crc32c(a.ctypes.data, a.nbytes))

    return crc


def load_golden_crc():
    out = []
    with open(os.path.join(ROOT, "tests", "golden", "rfc3720_crc32c.txt")) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            name, hx, crc = line.split()
            out.append((name, b"" if hx == "-" else bytes.fromhex(hx), int(crc, 16)))
    return out


def pytest_collection_modifyitems(config, items):
    # a hung GPU test must fail, not eat the whole gpurun budget
    for it in items:
        if it.get_closest_marker("gpu") and not it.get_closest_marker("timeout"):
            it.add_marker(pytest.mark.timeout(240))
