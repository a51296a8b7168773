"""The CPU oracle under AddressSanitizer + UndefinedBehaviorSanitizer (VERDICT r1 hygiene): the oracle
source is compiled with -fsanitize=address,undefined into tests/oracle_sanitize_driver.cpp, which drives
every entry-point family (declarations, scalar/array/batch maps with a rolled-back failing batch, device
slots, glue programs, coherence groups) in the default, literal-epoch and lenient modes."""
import os
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.skipif(shutil.which("g++") is None, reason="needs g++")
def test_oracle_under_asan_ubsan(tmp_path):
    exe = str(tmp_path / "oracle_sanitize")
    src = [os.path.join(ROOT, "tests", "oracle_sanitize_driver.cpp"), os.path.join(ROOT, "oracle", "cgcm_oracle.cpp")]
    subprocess.run(["g++", "-O1", "-g", "-std=c++17", "-ffp-contract=off", "-fsanitize=address,undefined",
                    "-fno-sanitize-recover=all", "-fno-omit-frame-pointer", "-o", exe] + src, check=True)
    env = dict(os.environ, ASAN_OPTIONS="detect_leaks=1:abort_on_error=1", UBSAN_OPTIONS="print_stacktrace=1")
    r = subprocess.run([exe], capture_output=True, text=True, env=env, timeout=300)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "oracle sanitize driver: ok" in r.stdout
