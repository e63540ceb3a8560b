"""Debug driver: the multi-GPU giant-kernel path on the loopback communicator."""
import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import numpy as np
import test_gpu_dist as T
import paper_conf_micro_chungnkk25_b200 as sr
import oracle as O
W = int(sys.argv[1]) if len(sys.argv) > 1 else 3
kid1 = np.zeros(5000, np.uint32)
t1 = (np.arange(5000) % 7 * 1000 + 5).astype(np.uint32)
st = []
got = T._dist_plan(sr, kid1, t1, 1, W, stats_out=st, z=T.Z95)
T.assert_plans_equal(got, O.plan(kid1, t1, 1, z=T.Z95))
print("ok", [s["owned_rows"] for s in st])
