"""Repeat the bench's C4 Jacobi measurement R times (variance check)."""
import json
import os
import sys
import types

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_temucinslsga24_b200 as pc  # noqa: E402
from paper_conf_sc_temucinslsga24_b200 import apps  # noqa: E402

args = types.SimpleNamespace(jacobi_n=int(os.environ.get("N", "16384")), jacobi_iters=int(os.environ.get("K", "50")))
torch.cuda.set_device(0)
for rep in range(int(os.environ.get("R", "4"))):
    r = bench.jacobi_bench(pc, apps, torch, args)
    print(json.dumps({k: (round(v["hbm_frac"], 3), round(v["us_per_iter"], 1)) for k, v in r.items() if isinstance(v, dict)}), flush=True)
