import sys, time; sys.path.insert(0, '.')
import paper_conf_pldi_eizenbergppmd17_b200 as bc
from bcgen.configs import ConfigPlan
for kw in (dict(n_blocks=6, tpb=64, iters=2, log2_buckets=5), dict(n_blocks=24, tpb=128, iters=2, log2_buckets=7),
           dict()):
    plan = ConfigPlan(6, bug=0, **kw)
    recs = plan.records()
    t = time.time()
    try:
        r = bc.detect(recs, plan.geometry, device="cuda:0")
        print(kw, len(recs), "status", r.status, len(r.races), round(time.time() - t, 2), flush=True)
    except Exception as e:
        print(kw, len(recs), "ERR", e, round(time.time() - t, 2), flush=True)
