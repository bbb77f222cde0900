"""One bc_detect on a config (for ncu: launches are numbered from the first detect)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import bench, paper_conf_pldi_eizenbergppmd17_b200 as bc
name = sys.argv[1] if len(sys.argv) > 1 else "c2"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 1
recs, geom, le, ce = bench.make_trace(name, bench.CONFIG_IDX.get(name, 2))
d = torch.from_numpy(recs.view(np.uint8)).cuda()
ctx = bc.Context(geom, device=0)
ctx.load_trace(d)
for _ in range(reps):
    st, stats = ctx.detect()
print(stats["kernel_launches"], stats["ms_kernel"], file=sys.stderr)
