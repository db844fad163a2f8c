"""GPU-side self-test of the parity harness (injected bugs must fail parity on the
GPU path, not only on the CPU one -- tests/test_oracle_pins.py covers that side).

Two kinds of injected bug, each of which the e_norm <= 1e-5 comparison against the FP64 oracle
must reject:
* plausible mistakes at the product boundary, made on the inputs of the real library: a bandwidth
  off by 1%, one source dropped, weights shifted by one row, targets shifted by one row, one
  coordinate axis mirrored;
* plausible kernel mistakes, made inside the kernels by the measurement build libks_dbg.so
  (`paper_conf_icppw_wangkbgj16_b200.build.build_debug`, work-dropping knobs that exist only with
  -DKS_DEBUG): two of the three split-FP16 products dropped, the weight ring reloaded once, the
  R = 1 epilogue math skipped, the V MMA skipped, a third of P never stored.  The same build with
  no knob set must pass, so the failures are the injected bugs and not the build.
"""
import os
import subprocess
import sys

import numpy as np
import pytest

import workloads
from tests.parity import TOL_3XTF32, e_norm

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icppw_wangkbgj16_b200 as ks  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def gpu(a, W, b, h, precision="auto"):
    with ks.KernelSum(a.shape[1], float(h), precision) as plan:
        plan.set_sources(torch.from_numpy(np.ascontiguousarray(a)).cuda(),
                         torch.from_numpy(np.ascontiguousarray(W)).cuda())
        V = plan.eval(torch.from_numpy(np.ascontiguousarray(b)).cuda())
        torch.cuda.synchronize()
    return V.cpu().numpy().astype(np.float64)


def rejected(err):
    return not (err <= TOL_3XTF32)  # NaN counts as rejected


@pytest.fixture(scope="module")
def case(oracle_mod):
    a, W, b, h = workloads.custom(3000, 700, 32, 4, 1.7, dist="gm", sigma=0.08, wkind="signed", seed=77)
    Vr = oracle_mod.oracle_eval(a, W, b, float(h))
    return a, W, b, h, Vr


def test_clean_passes(case):
    a, W, b, h, Vr = case
    assert e_norm(gpu(a, W, b, h), Vr, W) <= TOL_3XTF32


@pytest.mark.parametrize("bug", ["h_off_by_1pct", "drop_last_source", "weights_shifted", "targets_shifted",
                                 "axis_mirrored"])
def test_boundary_bugs_are_rejected(case, bug):
    a, W, b, h, Vr = case
    a2, W2, b2, h2 = a.copy(), W.copy(), b.copy(), float(h)
    if bug == "h_off_by_1pct":
        h2 = h2 * 1.01
    elif bug == "drop_last_source":
        a2, W2 = a2[:-1], W2[:-1]
    elif bug == "weights_shifted":
        W2 = np.roll(W2, 1, axis=0)
    elif bug == "targets_shifted":
        b2 = np.roll(b2, 1, axis=0)
    elif bug == "axis_mirrored":
        a2[:, 3] = 1.0 - a2[:, 3]
    err = e_norm(gpu(a2, W2, b2, h2), Vr, W)
    assert rejected(err), f"{bug}: e_norm {err:.3e} passed the 1e-5 bar"


@pytest.fixture(scope="module")
def dbg_lib():
    from paper_conf_icppw_wangkbgj16_b200 import build as b
    return b.build_debug(debug=1, prof=0, trace=0)


# (name, K, R, M, N, h / sqrt(K), environment knob, injected?).  Sizes: M = 65,536 gives every CTA
# more units than the weight ring has slots (the ring bug only shows after the first WS units); the
# one-product case uses few sources so its per-pair errors do not average out below the bar.
KERNEL_CASES = [
    ("r1_clean", 32, 1, 2600, 600, 0.3, {}, False),
    ("r1_no_epilogue_math", 32, 1, 2600, 600, 0.3, {"KS_R1_DEBUG": "1"}, True),
    ("rv_clean", 32, 8, 2600, 600, 0.3, {}, False),
    ("rv_no_v_mma", 32, 8, 2600, 600, 0.3, {"KS_RV_DEBUG": "1"}, True),
    ("rv_p_store_dropped", 32, 8, 2600, 600, 0.3, {"KS_RV_DEBUG": "32"}, True),
    ("tc_clean", 64, 16, 2600, 600, 0.3, {}, False),
    ("tc_clean_small", 64, 16, 48, 600, 0.15, {}, False),
    ("tc_one_split_product", 64, 16, 48, 600, 0.15, {"KS_TC_DEBUG_SKIP_V": "6"}, True),
    ("tc_clean_ring", 64, 2, 65536, 640, 0.3, {}, False),
    ("tc_weight_ring_once", 64, 2, 65536, 640, 0.3, {"KS_TC_DEBUG_SKIP_V": "4"}, True),
    ("tc_no_epilogue_math", 64, 2, 2600, 600, 0.3, {"KS_TC_DEBUG_SKIP_V": "1"}, True),
]


@pytest.mark.parametrize("name,K,R,M,N,hf,env,injected", KERNEL_CASES, ids=[c[0] for c in KERNEL_CASES])
def test_kernel_bugs_are_rejected(oracle_mod, dbg_lib, tmp_path, name, K, R, M, N, hf, env, injected):
    a, W, b, h = workloads.custom(M, N, K, R, hf * np.sqrt(K), dist="gm", sigma=0.08, wkind="signed", seed=K + R)
    src, out = tmp_path / "in.npz", tmp_path / "V.npy"
    np.savez(src, a=a, W=W, b=b, h=np.float64(h))
    e = dict(os.environ, KS_LIB=os.path.basename(dbg_lib), **env)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "tests", "gpu_child.py"), str(src), str(out), "auto"],
                       env=e, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    assert "libks_dbg.so" in r.stdout, r.stdout
    V = np.load(out)
    err = e_norm(V, oracle_mod.oracle_eval(a, W, b, float(h)), W)
    if injected:
        assert rejected(err), f"{name}: injected bug passed parity (e_norm {err:.3e})"
    else:
        assert err <= TOL_3XTF32, f"{name}: the measurement build without a knob fails parity ({err:.3e})"
