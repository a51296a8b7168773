"""The general per-chunk code of the two pipelined passes (fwd_chunk_slow, rev_chunk_slow in
csrc/kernels.cu) against the oracle on its own.

k_fwd_fast / k_rev_fast send only the chunks with a NULL, a miss, an activation, a ragged end, a
copy-back and the like through that code; calls of 2^31 chunks or more (32 GiB of slots) run every chunk
through it (k_fwd_big / k_rev_big).  CGCM_FORCE_BIG selects the latter for every call, so this test
re-runs the modules that exercise the hot passes (page-directory lookup cases, deferred references,
device-array parity programs) in a child process with it set: every chunk of every call then takes the
general code, and each call is still compared with the oracle (Alg. 1-3).
"""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_hot_passes_with_every_chunk_on_the_general_path():
    env = dict(os.environ, CGCM_FORCE_BIG="1")
    cmd = [sys.executable, "-m", "pytest", "-x", "-q", "-m", "gpu", "-p", "no:cacheprovider",
           "tests/test_gpu_pagedir.py", "tests/test_gpu_deferred.py",
           "tests/test_gpu_parity.py", "-k", ("pagedir or (deferred and not rewritten) or config_C_device or shadow_fallback or ragged or permutation "
                  "or compact_word or 4GiB or epoch_origin or (random_device_slices and auto and not churn and not lenient)")]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=1500)
    tail = (r.stdout + r.stderr)[-3000:]
    assert r.returncode == 0, tail
    assert " passed" in r.stdout, tail
