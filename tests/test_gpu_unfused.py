"""NEXT-1 comparison design on the GPU (tools/unfused.py): cuBLAS SGEMM writes the
target x source block to HBM, one kernel (tools/unfused_expw.cu) reads it once (norms,
d^2 >= 0 clamp, exp2, times W, row sums).  It must compute the same V as the oracle and
as the eager multi-pass version, so the fused/unfused speed and DRAM comparison
(SS7) compares equal results."""
import os
import sys

import numpy as np
import pytest

import workloads
from tests.parity import TOL_FP32, e_norm

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
from unfused import unfused_eval  # noqa: E402


@pytest.mark.parametrize("K,R,M,N,wkind", [(32, 1, 3001, 700, "pos"), (8, 1, 4096, 999, "pos"),
                                             (64, 3, 1500, 300, "signed"), (256, 16, 900, 200, "signed")])
def test_one_pass_unfused_matches_oracle(oracle_mod, K, R, M, N, wkind):
    a, W, b, h = workloads.custom(M, N, K, R, 0.3 * np.sqrt(K), wkind=wkind, seed=K * 7 + R)
    ta, tw, tb = (torch.from_numpy(x).cuda() for x in (a, W, b))
    Vp = unfused_eval(ta, tw, tb, float(h), mode="pass", budget_bytes=4 * M * 128).cpu().numpy()  # chunked
    Ve = unfused_eval(ta, tw, tb, float(h), mode="eager").cpu().numpy()
    Vr = oracle_mod.oracle_eval(a, W, b, float(h))
    assert e_norm(Vp, Vr, W) <= TOL_FP32
    assert e_norm(Ve, Vr, W) <= TOL_FP32
