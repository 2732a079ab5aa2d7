"""Host-side checks of the benchmark plumbing that need no GPU: the reference
arm's JSON line (the CPU oracle, per the tier rules) and the product's host
helper that turns a split into block times (used for the f2 workload), checked
against the oracle's own block statistics."""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle
from paper_conf_icpp_luoyww0023_b200 import workloads as wl

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                        "--warmup", "1"], capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    d = json.loads(r.stdout.strip().splitlines()[-1])
    assert d["impl"] == "reference" and d["unit"] == "evals/s" and d["higher_is_better"] is True
    assert d["value"] > 0 and d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]


def test_reference_arm_other_ranks_exit_quietly():
    env = dict(os.environ, RANK="1", WORLD_SIZE="2", LOCAL_RANK="1")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                        "--warmup", "1"], capture_output=True, text=True, timeout=600, cwd=ROOT, env=env)
    assert r.returncode == 0 and r.stdout.strip() == ""


def test_block_times_match_oracle_statistics():
    # split_block_times (C ABI, host only) against the oracle's exact block statistics
    import importlib
    split = importlib.import_module("paper_conf_icpp_luoyww0023_b200.split")
    lat, ovh = wl.chain("resnet50_122")
    pop = wl.sparse_population(len(lat), 64, seed=5)
    for row in pop:
        b = split.split_block_times(lat, ovh, row)
        st = oracle.fitness(lat, ovh, row)
        assert len(b) == st["k"]
        assert sum(b) == st["s1"] and sum(x * x for x in b) == st["s2"]
        assert sum(b) - int(np.sum(lat)) == st["overhead"]


def test_block_times_edges_and_errors():
    import importlib
    split = importlib.import_module("paper_conf_icpp_luoyww0023_b200.split")
    lat = np.array([3, 4, 5], dtype=np.int64)
    assert split.split_block_times(lat, None, np.array([0], np.uint64)) == [12]           # unsplit
    assert split.split_block_times(lat, [7, 9], np.array([0b11], np.uint64)) == [3, 11, 14]
    assert split.split_block_times(lat, [7, 9], np.array([0b111 | (1 << 63)], np.uint64)) == [3, 11, 14]  # padding
    with pytest.raises(split.SplitError) as e:
        split.split_block_times(np.array([1, -1]), None, np.array([1], np.uint64))
    assert e.value.code == split.SPLIT_E_INVAL
    import ctypes as C
    k = C.c_uint32(0)
    out = np.zeros(1, np.int64)
    rc = split.lib().split_block_times(lat.ctypes.data_as(C.c_void_p), None, 3,
                                        np.array([0b11], np.uint64).ctypes.data_as(C.c_void_p),
                                        out.ctypes.data_as(C.c_void_p), 1, C.byref(k))
    assert rc == split.SPLIT_E_RANGE and k.value == 3 and out[0] == 3
