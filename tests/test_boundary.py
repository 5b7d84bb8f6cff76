"""The C-ABI library loads without a GPU and exports every function include/*.h declares."""
import ctypes
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    names = set()
    for h in ("orion.h", "orion_kernels.h"):
        src = open(os.path.join(ROOT, "include", h)).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        for m in re.finditer(r"^\s*(?:const\s+)?[a-z_0-9]+\s*\*?\s*(orion_[a-z_0-9]+)\s*\(", src, flags=re.M):
            names.add(m.group(1))
    return names


def test_exports_every_declared_symbol():
    from paper_conf_eurosys_stratimk24_b200 import _lib
    names = _declared()
    assert len(names) >= 20, names
    out = subprocess.check_output(["nm", "-D", "--defined-only", _lib.LIB_PATH]).decode()
    exported = {l.split()[-1] for l in out.splitlines() if " T " in l}
    missing = names - exported
    assert not missing, missing
    for n in names:
        getattr(_lib.lib, n)


def test_no_libcuda_link_dependency():
    """liborion must load on a driverless host (resolves driver entry points at run time)."""
    from paper_conf_eurosys_stratimk24_b200 import _lib
    out = subprocess.check_output(["ldd", _lib.LIB_PATH]).decode()
    assert "libcuda.so" not in out and "libtorch" not in out


def test_kernel_table_names():
    from paper_conf_eurosys_stratimk24_b200 import _lib
    import re
    names = _lib.kernel_names()
    hdr = open(os.path.join(ROOT, "include", "orion_kernels.h")).read()
    enum = {int(v): k.lower() for k, v in re.findall(r"ORION_FN_(\w+) = (\d+)", hdr) if k != "COUNT"}
    count = int(re.search(r"ORION_FN_COUNT = (\d+)", hdr).group(1))
    assert len(names) == count == len(enum)
    assert [enum[i] for i in range(count)] == names


def test_cuda_backend_fails_cleanly_without_gpu():
    import torch
    if torch.cuda.is_available():
        return
    from paper_conf_eurosys_stratimk24_b200 import _lib, Orion
    try:
        Orion(backend=_lib.BACKEND_CUDA)
    except _lib.OrionError as e:
        assert e.code in (_lib.E_NODEV, _lib.E_CUDA)
    else:
        raise AssertionError("CUDA backend created without a GPU")


def test_record_layouts():
    from paper_conf_eurosys_stratimk24_b200 import _lib
    assert ctypes.sizeof(_lib.Op) == 224
    assert ctypes.sizeof(_lib.Config) == 80
