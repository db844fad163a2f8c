"""One step of the fused design (ks_set_sources + ks_eval through libks.so) or of the unfused
comparison design (tools/unfused.py: cuBLAS SGEMM + one-pass kernel) on a BASELINE config, the
measured step inside an NVTX range "measured" so ncu profiles exactly its kernels:

    ncu --nvtx --nvtx-include "measured/" --metrics gpu__time_duration.sum,dram__bytes_read.sum,\\
        dram__bytes_write.sum,lts__t_bytes.sum --csv --log-file fused.csv python tools/fig8_step.py fused
    python tools/fig8.py fused.csv unfused.csv --md profiles/<round>/fig8.md
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import torch  # noqa: E402

import paper_conf_icppw_wangkbgj16_b200 as ks  # noqa: E402
import workloads  # noqa: E402
from unfused import unfused_eval  # noqa: E402

design = sys.argv[1]
cfg = int(sys.argv[2]) if len(sys.argv) > 2 else 3
a, W, b, h = workloads.make(cfg)
ta, tw, tb = (torch.from_numpy(x).cuda() for x in (a, W, b))
plan = ks.KernelSum(a.shape[1], float(h))
V = torch.empty((b.shape[0], W.shape[1]), device="cuda")


def step():
    if design == "fused":
        plan.set_sources(ta, tw)
        plan.eval(tb, out=V)
    else:
        V.copy_(unfused_eval(ta, tw, tb, float(h)))


step()
torch.cuda.synchronize()
torch.cuda.nvtx.range_push("measured")
step()
torch.cuda.synchronize()
torch.cuda.nvtx.range_pop()
print(design, "done")
