"""Quick check of one warp-specialized configuration against the classic in-plane kernel
(bit-identical by construction) on a small grid.  Run under `timeout`."""
import sys
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import stencil_inputs as si
import paper_conf_ipps_tangtkwkgtw13_b200 as S

n, r = int(sys.argv[1]) if len(sys.argv) > 1 else 70, 4
cfgs = [dict(kernel="inplane", tx=16, ty=4, rx=4, ry=4, stages=4, zsegs=2, zbox=2),
        dict(kernel="inplane_ws", tx=16, ty=4, rx=4, ry=2, stages=3, zsegs=2, zbox=2),
        dict(kernel="inplane_ws", tx=16, ty=16, rx=4, ry=4, stages=4, zsegs=2, zbox=2),
        dict(kernel="inplane_ws", tx=32, ty=7, rx=4, ry=2, stages=4, zsegs=1, zbox=4)]
with S.Plan(n, n - 7, n + 3, r, si.coeffs_as("heat", r, "f32"), "f32") as p:
    a, b = p.alloc(), p.alloc()
    p.fill_counter(a, 3)
    ref = None
    for c in cfgs:
        p.set_config(**c)
        p.run(a, b, 3)
        torch.cuda.synchronize()
        print(c, "ok", flush=True)
        if ref is None:
            ref = b.clone()
        else:
            print("  bit-identical to inplane:", bool(torch.equal(ref, b)), flush=True)
