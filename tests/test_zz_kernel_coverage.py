"""Every kernel in libsg.so is exercised by the GPU parity tests.

Runs last (file order) in the same pytest process as the other `-m gpu` tests: libsg records every distinct
kernel it launches (sg_launched_kernels, test instrumentation); this test lists the entry kernels the library
contains (cuobjdump -symbols: STO_ENTRY, minus the CUB library's) and requires each of them to have been
launched by the preceding parity tests.  Only meaningful for the full GPU suite (skipped under -k).
"""
import re
import shutil
import subprocess

import pytest

from conftest import gpu_available

pytestmark = [pytest.mark.gpu, pytest.mark.skipif(not gpu_available(), reason="needs a CUDA device")]


def library_kernels(path):
    exe = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    out = subprocess.run([exe, "-symbols", path], capture_output=True, text=True).stdout
    names = set()
    for line in out.splitlines():
        f = line.split()
        if len(f) >= 4 and f[0] == "STT_FUNC" and "STO_ENTRY" in f and not f[-1].startswith("_ZN3cub"):
            names.add(f[-1])
    return names


def test_every_library_kernel_was_launched(request):
    if request.config.option.keyword or (request.config.option.markexpr or "") != "gpu":
        pytest.skip("needs the full `pytest -m gpu` run")
    from paper_conf_ppopp_murarasuwbbp11_b200 import _sg
    kernels = library_kernels(_sg.LIB_PATH)
    launched = set(_sg.sg_launched_kernels())
    assert kernels, "no kernels found in the library"
    missing = sorted(k for k in kernels if k not in launched)
    assert not missing, "kernels never launched by the parity tests:\n" + "\n".join(missing)
