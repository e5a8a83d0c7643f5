import sys, time
import tdfs_inputs as T, oracle as O
import paper_conf_icde_yuan0ha0024_b200 as M
from tests import gpu_util as U
g = T.rmat(9, 8, 5)
q = T.query(sys.argv[1])
order = O.oracle_order(q)
kw = eval("dict(" + sys.argv[2] + ")")
t = time.time()
print(sys.argv[1], kw, U.count(g, q, "auto", order=order, stats=True, **kw), O.count(g, q, "auto", order=order), time.time() - t, flush=True)
