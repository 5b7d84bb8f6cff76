"""ctypes access to oracle/liboracle_policy.so (CPU oracle; tests and bench cpu_baseline only)."""
import ctypes
import os
import subprocess

ORACLE_DIR = os.path.dirname(os.path.abspath(__file__))
_lib = None


def lib():
    global _lib
    if _lib is None:
        so = os.path.join(ORACLE_DIR, "liboracle_policy.so")
        src = os.path.join(ORACLE_DIR, "policy.c")
        if not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
            subprocess.check_call(["make", "-s", "-C", ORACLE_DIR])
        _lib = ctypes.CDLL(so)
        _lib.oracle_replay.argtypes = [ctypes.c_char_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_size_t,
                                       ctypes.POINTER(ctypes.c_size_t)]
        _lib.oracle_brute.argtypes = [ctypes.c_char_p, ctypes.c_size_t, ctypes.c_uint64,
                                      ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64),
                                      ctypes.c_char_p, ctypes.c_size_t]
    return _lib


def replay(log: bytes) -> bytes:
    """Return the decision section (u64 n + 32-byte records) the oracle derives from log's tape."""
    L = lib()
    need = ctypes.c_size_t(0)
    r = L.oracle_replay(log, len(log), None, 0, ctypes.byref(need))
    if r not in (0, -20):
        raise RuntimeError(f"oracle_replay failed: {r}")
    buf = ctypes.create_string_buffer(need.value)
    r = L.oracle_replay(log, len(log), buf, need.value, ctypes.byref(need))
    if r != 0:
        raise RuntimeError(f"oracle_replay failed: {r}")
    return buf.raw[:need.value]


def brute(hdr: bytes, max_nodes=0):
    L = lib()
    paths, nodes = ctypes.c_uint64(0), ctypes.c_uint64(0)
    err = ctypes.create_string_buffer(256)
    r = L.oracle_brute(hdr, len(hdr), max_nodes, ctypes.byref(paths), ctypes.byref(nodes), err, 256)
    if r < 0:
        raise RuntimeError(f"oracle_brute parse error {r}")
    return r, paths.value, nodes.value, err.value.decode()
