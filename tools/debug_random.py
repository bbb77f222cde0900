"""Debug helper: run GPU vs oracle on random traces, save mismatching traces to gpurun_out/."""
import os, sys, numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle, paper_conf_pldi_eizenbergppmd17_b200 as bc
from bcgen.fuzz import random_trace
os.makedirs("gpurun_out/dbg", exist_ok=True)
bad = 0
for seed in range(int(sys.argv[1]), int(sys.argv[2])):
    recs, tb = random_trace(seed)
    geom = tb.geom.as_dict()
    st, want, _ = oracle.detect_geom(recs, geom)
    try:
        res = bc.detect(recs, geom)
        got, gst = res.races, res.status
    except bc.BcError as e:
        got, gst = None, e.status
    ok = gst == st and got is not None and len(got) == len(want) and np.array_equal(got.view(np.uint8), want.view(np.uint8))
    if not ok:
        bad += 1
        np.save(f"gpurun_out/dbg/seed{seed}_recs.npy", recs)
        if got is not None:
            np.save(f"gpurun_out/dbg/seed{seed}_gpu.npy", got)
        print("MISMATCH seed", seed, "status", gst, st, "n", None if got is None else len(got), len(want), geom, flush=True)
print("bad", bad)
