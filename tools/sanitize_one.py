"""Small bc_detect workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
C1, random traces (one window and many), a reduced C4 and C2, values, the warp-size re-split and a
2-rank block-sharded run -- each checked against the oracle."""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np
import bcgen, oracle
import paper_conf_pldi_eizenbergppmd17_b200 as bc
from bcgen.configs import ConfigPlan
from bcgen.fuzz import random_trace, random_values


def same(recs, geom, **kw):
    st, want, _ = oracle.detect_geom(recs, geom, values=kw.get("values"))
    res = bc.detect(recs, geom, device="cuda:0", **kw)
    assert res.status == st, (res.status, st)
    assert st != 0 or np.array_equal(res.races.view(np.uint8), want.view(np.uint8))


recs, tb = bcgen.configs.make_c1()
same(recs, tb.geom.as_dict())
for seed in range(3):
    recs, tb = random_trace(seed)
    same(recs, tb.geom.as_dict())
    same(recs, tb.geom.as_dict(), window_events=64)
recs, tb = random_trace(7, same_value=True, n_glob=2)
same(recs, tb.geom.as_dict(), values=random_values(recs, 7))
for cfg, kw in [(4, dict(n_blocks=12, log2_nodes=14, nodes_per_thread=2, inj_scale=4)), (2, dict(n_blocks=4, iters=3))]:
    p = ConfigPlan(cfg, **kw)
    same(p.records(), p.geometry)
    same(p.records(), p.geometry, window_events=2000)
recs, tb = random_trace(11)
d, g2, org = bc.split_warps(recs, tb.geom.as_dict(), 8)
from test_shard import assert_sharded
p = ConfigPlan(4, n_blocks=12, log2_nodes=14, nodes_per_thread=2, inj_scale=4)
assert_sharded(p.records(), p.geometry, 2)
# the sampled page set misses a page written by middle lanes only: K4 flags it, the detect re-runs
from bcgen import GLOBAL_BASE, TraceBuilder
tb = TraceBuilder(grid=(2, 1, 1), block=(32, 1, 1))
tb.st(tb.warp(0), lambda l: GLOBAL_BASE + (0 if l in (0, 31) else 5 << 20) + 4 * l)
tb.ld(tb.warp(1), lambda l: GLOBAL_BASE + (5 << 20) + 4 * l)
same(tb.records(), tb.geom.as_dict())
print("sanitize workload ok")
