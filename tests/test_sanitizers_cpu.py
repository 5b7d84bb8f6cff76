"""SURVEY §4 T6 on the host side: liborion's scheduler, SPSC rings, native client drivers and the
FAKE backend's stream threads built with ThreadSanitizer (and separately AddressSanitizer +
UndefinedBehaviorSanitizer) and driven by tools/tsan/sched_driver.cpp with concurrent HP / BE
producers under several policy readings. Any sanitizer report fails the test."""
import os
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_eurosys_stratimk24_b200", "csrc")


def _build(tmp_path, san):
    exe = str(tmp_path / f"sched_{san.replace(',', '_')}")
    cmd = ["g++", "-std=c++17", "-O1", "-g", f"-fsanitize={san}", "-fno-omit-frame-pointer", "-pthread",
           "-I" + os.path.join(ROOT, "include"), "-I" + CSRC,
           os.path.join(CSRC, "orion_core.cpp"), os.path.join(CSRC, "backend_fake.cpp"),
           os.path.join(ROOT, "tools", "tsan", "sched_driver.cpp"), "-o", exe]
    subprocess.check_call(cmd)
    return exe


@pytest.mark.skipif(shutil.which("g++") is None, reason="no g++")
@pytest.mark.parametrize("san", ["thread", "address,undefined"])
def test_scheduler_under_sanitizer(san, tmp_path):
    exe = _build(tmp_path, san)
    env = dict(os.environ, TSAN_OPTIONS="halt_on_error=1 exitcode=66 second_deadlock_stack=1",
               ASAN_OPTIONS="halt_on_error=1 detect_leaks=1", UBSAN_OPTIONS="halt_on_error=1 print_stacktrace=1")
    for flags in ("0", "3", "31", "448"):
        p = subprocess.run([exe, flags], capture_output=True, text=True, timeout=300, env=env)
        assert p.returncode == 0, (flags, p.returncode, p.stdout[-2000:], p.stderr[-4000:])
        assert "Sanitizer" not in p.stderr and "runtime error" not in p.stderr, p.stderr[-4000:]
