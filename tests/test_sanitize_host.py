"""Host sanitizers: the C oracle and the C generators built with
AddressSanitizer + UndefinedBehaviorSanitizer and run over small and edge-case inputs
by tests/native/sanitize_driver.c.  Any out-of-bounds access, use after free, signed
overflow or misaligned access aborts the driver with a report."""
import os
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.skipif(shutil.which("gcc") is None, reason="needs gcc")
def test_oracle_and_generators_under_asan_ubsan(tmp_path):
    exe = str(tmp_path / "sanitize_driver")
    subprocess.check_call(
        ["gcc", "-O1", "-g", "-fsanitize=address,undefined", "-fno-sanitize-recover=all",
         "-fno-omit-frame-pointer", "-ffp-contract=off",
         os.path.join(ROOT, "tests", "native", "sanitize_driver.c"),
         os.path.join(ROOT, "oracle", "oracle.c"), os.path.join(ROOT, "gen", "gen.c"),
         "-o", exe, "-lm"])
    env = dict(os.environ, ASAN_OPTIONS="detect_leaks=0:abort_on_error=1",
               UBSAN_OPTIONS="print_stacktrace=1:halt_on_error=1")
    r = subprocess.run([exe], capture_output=True, text=True, env=env, timeout=600)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "sanitize driver ok" in r.stdout
