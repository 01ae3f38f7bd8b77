"""The seeded generators: deterministic, thread-count independent, canonical CSR."""
import hashlib
import os
import subprocess
import sys

import numpy as np
import pytest

import datagen
from datagen import configs

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _canonical(M, K, rp, ci):
    assert rp[0] == 0 and rp[-1] == len(ci) and np.all(np.diff(rp) >= 0)
    assert len(ci) == 0 or (ci.min() >= 0 and ci.max() < K)
    d = np.diff(ci.astype(np.int64))
    rows = np.repeat(np.arange(M), np.diff(rp))
    same_row = rows[1:] == rows[:-1]
    assert np.all(d[same_row] > 0)


@pytest.mark.parametrize("name", ["c1", "c2"])
def test_config_pattern_canonical_and_shaped(name):
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    _canonical(cfg.M, cfg.K, rp, ci)
    assert abs(len(ci) - cfg.nnz) / cfg.nnz < 0.01
    assert np.diff(rp).max() <= cfg.d_max


def test_banded_small():
    rp, ci = datagen.banded_csr(5005, 5005, 40, 64, 2, 3000, 4)
    _canonical(5005, 5005, rp, ci)
    deg = np.diff(rp)
    assert sorted(deg)[-2:] == [3000, 3000]
    rows = np.repeat(np.arange(5005), deg)
    normal = deg[rows] == 40
    assert np.all(np.abs(ci[normal].astype(np.int64) - rows[normal]) <= 64)


def _hash_c2(threads):
    code = ("import hashlib,sys; sys.path.insert(0, %r); from datagen import configs;"
            "c=configs.get('c2'); rp,ci=configs.make_pattern(c); v=configs.make_values(c,len(ci));"
            "print(hashlib.sha1(rp.tobytes()+ci.tobytes()+v.tobytes()).hexdigest())") % ROOT
    env = dict(os.environ, OMP_NUM_THREADS=str(threads))
    return subprocess.check_output([sys.executable, "-c", code], env=env).decode().strip()


def test_thread_count_independent():
    assert _hash_c2(1) == _hash_c2(4)


def test_values_deterministic():
    a = datagen.uniform(1, 2, 1000)
    b = datagen.uniform(1, 2, 1000)
    c = datagen.uniform(1, 3, 1000)
    assert np.array_equal(a, b) and not np.array_equal(a, c)
    assert a.min() >= -1 and a.max() < 1
    i = datagen.integers(1, 2, 10000)
    assert set(np.unique(i).tolist()) == set(range(-4, 5))
    d = datagen.dyadic(1, 2, 10000)
    assert np.all(d * 8 == np.round(d * 8))
