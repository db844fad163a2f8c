"""The unfused comparison design (tools/unfused.py, NEXT-1) computes the same
V as the oracle (CPU tensors here; bench.py --impl unfused runs it on the GPU)."""
import os
import sys

import numpy as np
import pytest

import workloads
from tests.parity import TOL_FP32, e_norm

torch = pytest.importorskip("torch")
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
from unfused import hbm_bytes_per_pair, unfused_eval  # noqa: E402


@pytest.mark.parametrize("K,R,wkind", [(8, 1, "pos"), (32, 1, "signed"), (20, 3, "pos")])
def test_unfused_matches_oracle(oracle_mod, K, R, wkind):
    a, W, b, h = workloads.custom(700, 300, K, R, 0.3 * np.sqrt(K), wkind=wkind, seed=K + R)
    V = unfused_eval(torch.from_numpy(a), torch.from_numpy(W), torch.from_numpy(b), float(h),
                     budget_bytes=4 * 700 * 64).numpy()          # forces 5 target chunks
    Vr = oracle_mod.oracle_eval(a, W, b, float(h))
    assert e_norm(V, Vr, W) <= TOL_FP32


def test_unfused_traffic_model():
    t = hbm_bytes_per_pair()
    assert t["best_unfused"] == 8 and t["eager_passes"] > t["best_unfused"]
