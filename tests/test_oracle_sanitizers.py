"""The CPU oracle under AddressSanitizer + UndefinedBehaviorSanitizer (SURVEY §5 aux: ASan/UBSan on
the oracle).  Builds oracle/gbdt_oracle.c with a standalone driver (oracle/sanitize/driver.c) and
runs it: Table I, seeded random matrices with NaN-missing values and repeated values, follow mode,
prediction.  Any memory error or undefined behaviour aborts with a non-zero status."""
import os
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.skipif(shutil.which("gcc") is None, reason="needs gcc")
def test_oracle_clean_under_asan_ubsan(tmp_path):
    exe = tmp_path / "orc_san"
    src = [os.path.join(ROOT, "oracle", "gbdt_oracle.c"), os.path.join(ROOT, "oracle", "sanitize", "driver.c")]
    subprocess.check_call(["gcc", "-O1", "-g", "-std=c11", "-fno-omit-frame-pointer", "-ffp-contract=off",
                           "-fsanitize=address,undefined", "-fno-sanitize-recover=all", *src, "-o", str(exe), "-lm"])
    env = dict(os.environ, ASAN_OPTIONS="detect_leaks=1:abort_on_error=1", UBSAN_OPTIONS="print_stacktrace=1")
    r = subprocess.run([str(exe)], capture_output=True, text=True, env=env, timeout=600)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "rc=0" in r.stdout
