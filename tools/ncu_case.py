"""One in-plane sweep configuration of a 512^3 grid, for an ncu capture.

    python tools/ncu_case.py f64 4 --tune            # prints the tuned config as JSON
    ncu --set full -k regex:inplane_sweep -s 2 -c 1 -o out python tools/ncu_case.py f64 4 '<json>'
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import stencil_inputs as si  # noqa: E402
import paper_conf_ipps_tangtkwkgtw13_b200 as S  # noqa: E402

dtype, r = sys.argv[1], int(sys.argv[2])
n = 512
with S.Plan(n, n, n, r, si.coeffs_as("heat", r, dtype), dtype) as p:
    a, b = p.alloc(), p.alloc()
    p.fill_counter(a, 3)
    if sys.argv[3] == "--tune":
        s0, s1 = p.alloc(), p.alloc()
        s0.copy_(a)
        s1.copy_(a)
        p.tune(kernel="inplane", beta=5, iters_per_rep=2, reps=2, scratch=(s0, s1))
        print(json.dumps(p.config))
    else:
        p.set_config(**json.loads(sys.argv[3]))
        p.run(a, b, 4)
        torch.cuda.synchronize()
