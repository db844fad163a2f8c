"""Child process of tests/test_gpu_harness.py: evaluates one case through the library KS_LIB
selects (the measurement build libks_dbg.so with a work-dropping knob in the environment) and
saves V.  Usage: python tests/gpu_child.py <inputs.npz> <out.npy> <precision>"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_icppw_wangkbgj16_b200 as ks  # noqa: E402


def main():
    src, out, prec = sys.argv[1], sys.argv[2], sys.argv[3]
    d = np.load(src)
    a, W, b, h = d["a"], d["W"], d["b"], float(d["h"])
    with ks.KernelSum(a.shape[1], h, prec) as plan:
        plan.set_sources(torch.from_numpy(a).cuda(), torch.from_numpy(W).cuda())
        V = plan.eval(torch.from_numpy(b).cuda())
        torch.cuda.synchronize()
        info = plan.info()
    np.save(out, V.cpu().numpy().astype(np.float64))
    print("kernel", info["kernel"], "lib", os.path.basename(ks.LIB_PATH), flush=True)


if __name__ == "__main__":
    main()
