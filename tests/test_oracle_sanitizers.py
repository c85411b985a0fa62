"""Host sanitizers on the oracle ("host ASan/UBSan build of csrc/ and oracle/"): oracle.c built with
-fsanitize=address,undefined (errors fatal), loaded through ORACLE_LIB in a subprocess that preloads the ASan
runtime, runs the oracle's pin tests.  Any out-of-bounds access, use-after-free, signed overflow or misaligned
access in the oracle aborts the subprocess.  (The CUDA library's device code is covered by compute-sanitizer:
scripts/sanitize.sh, profiles/r1_sanitizers.txt; its host side by tests/test_abi.py's ASan load below.)"""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _asan_runtime():
    r = subprocess.run(["gcc", "-print-file-name=libasan.so"], capture_output=True, text=True)
    p = r.stdout.strip()
    return p if os.path.isabs(p) and os.path.exists(p) else None


@pytest.fixture(scope="module")
def sanitized_oracle(tmp_path_factory):
    rt = _asan_runtime()
    if rt is None:
        pytest.skip("no ASan runtime")
    out = str(tmp_path_factory.mktemp("asan") / "liboracle_asan.so")
    subprocess.check_call(["gcc", "-O1", "-g", "-fno-omit-frame-pointer", "-fsanitize=address,undefined",
                           "-fno-sanitize-recover=all", "-fopenmp", "-shared", "-fPIC", "-std=gnu11",
                           os.path.join(ROOT, "oracle", "oracle.c"), "-o", out, "-lm"])
    return out, rt


def test_oracle_pins_under_asan_ubsan(sanitized_oracle):
    lib, rt = sanitized_oracle
    env = {**os.environ, "ORACLE_LIB": lib, "LD_PRELOAD": rt, "OMP_NUM_THREADS": "4",
           "ASAN_OPTIONS": "detect_leaks=0:abort_on_error=1", "UBSAN_OPTIONS": "print_stacktrace=1:halt_on_error=1"}
    tests = [os.path.join(ROOT, "tests", f) for f in
             ("test_oracle_spmm.py", "test_oracle_perm.py", "test_oracle_features.py", "test_oracle_features_b200.py",
              "test_oracle_misc.py")]
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider", "-m", "not gpu",
                        "-k", "not bruteforce_large", *tests], cwd=ROOT, env=env, capture_output=True, text=True,
                       timeout=900)
    assert r.returncode == 0, (r.stdout[-3000:], r.stderr[-3000:])
    assert "passed" in r.stdout
    # the subprocess really ran the sanitized build (mapped, with the ASan runtime)
    chk = ("import oracle, synthetic as syn; a = syn.rmat(8, 4, 1); oracle.permute(a, 'cta_aware'); "
           "m = open('/proc/self/maps').read(); print('asan' if 'liboracle_asan' in m and 'libasan' in m else 'plain')")
    r = subprocess.run([sys.executable, "-c", chk], cwd=ROOT, env=env, capture_output=True, text=True, timeout=300)
    assert r.stdout.strip().endswith("asan"), (r.stdout, r.stderr[-2000:])


def test_asan_catches_an_overflow(sanitized_oracle, tmp_path):
    """The harness is live: a planted out-of-bounds read (a rowidx one entry short) aborts under ASan."""
    lib, rt = sanitized_oracle
    env = {**os.environ, "ORACLE_LIB": lib, "LD_PRELOAD": rt, "ASAN_OPTIONS": "detect_leaks=0"}
    bad = ("import numpy as np, oracle, synthetic as syn; a = syn.rmat(8, 4, 1); "
           "r = a.rowidx[:-1].copy(); "
           "oracle._load().oracle_features(a.M, a.N, r.ctypes.data, a.colidx.ctypes.data, None, 32, 32, 32, "
           "np.zeros(24).ctypes.data)")
    r = subprocess.run([sys.executable, "-c", bad], cwd=ROOT, env=env, capture_output=True, text=True, timeout=300)
    assert r.returncode != 0 and "AddressSanitizer" in r.stderr, r.stderr[-1500:]
