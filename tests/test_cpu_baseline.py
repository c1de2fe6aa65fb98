"""Tuned parallel CPU C2R (cpu_baseline/) against the oracle's definition,
bit-exact.  It is a bench baseline only; these tests keep it honest.

The checks run in a child interpreter: the OpenMP thread pool must not live in the pytest
process, which later forks gloo workers (tests/test_dist_cpu.py)."""
import os
import subprocess
import sys

from conftest import ROOT

CHECK = r'''
import numpy as np, oracle, workloads, cpu_baseline as cb
for eb in (4, 8):
    for m, n in workloads.small_shapes(24):
        X = workloads.random_words(m * n, eb, seed=m * 64 + n)
        Y = X.copy(); cb.c2r(Y, m, n)
        assert Y.tobytes() == oracle.transpose(X, m, n).tobytes(), (m, n, eb)
for m, n in [(1200, 1800), (1800, 1200), (333, 4097), (4096, 300), (1000, 1000)]:
    X = workloads.random_words(m * n, 4, seed=m ^ n)
    Y = X.copy(); cb.c2r(Y, m, n)
    assert Y.tobytes() == oracle.transpose(X, m, n).tobytes(), (m, n)
print("cpu_baseline ok")
'''


def test_tuned_cpu_c2r_matches_oracle():
    r = subprocess.run([sys.executable, "-c", CHECK], cwd=ROOT, capture_output=True, text=True, timeout=600,
                       env=dict(os.environ, PYTHONPATH=ROOT))
    assert r.returncode == 0 and "cpu_baseline ok" in r.stdout, r.stderr[-2000:]
