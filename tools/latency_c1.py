import sys, time
sys.path.insert(0, '.')
import seqgen, numpy as np
from paper_conf_ipps_mendoncam13_b200 import Database
w = seqgen.make_workload("C1")
D = Database(w.db)
for k in range(3): D.search(w.queries, top_k=10)
ts=[]
for k in range(20):
    t=time.perf_counter(); r=D.search(w.queries, top_k=10); ts.append(time.perf_counter()-t)
print("C1 host latency ms: median %.3f min %.3f  device %.3f ms  units %d launches %d" % (1e3*np.median(ts), 1e3*min(ts), 1e3*r.stats['seconds_device'], r.stats['n_units'], r.stats['kernel_launches']))
ts=[]
for k in range(20):
    t=time.perf_counter(); r=D.search(w.queries, top_k=10, outputs_on_device=True); ts.append(time.perf_counter()-t)
print("C1 device-out latency ms: median %.3f" % (1e3*np.median(ts)))
