import sys, time, numpy as np
sys.path.insert(0,'.')
from synth import configs as C
from paper_conf_ipps_tianmyd20_b200 import _lib as L
w=C.PL32M; t=time.time(); g=C.graph(w); print('gen', time.time()-t, flush=True)
rows=np.repeat(np.arange(g.n, dtype=np.int32), np.diff(g.rowptr))
for sw in [10, 30]:
    t=time.time()
    pl=L.Plan(g.n, g.rowptr, g.col, w.P, 0.0657, build_device=False, lp_sweeps=sw)
    st=pl.stats(); perm=pl.perm()
    pos=np.empty(g.n, np.int32); pos[perm]=np.arange(g.n, dtype=np.int32)
    d=np.abs(pos[rows].astype(np.int64)-pos[g.col])
    print(sw, 'sweeps', st['lp_sweeps'], 'clusters', st['clusters'], 'intra', st['intra_edges']/st['nnz'], 'near(<32K)', (d<32768).mean(), 'near(<128K)', (d<131072).mean(), 'near(<512K)', (d<524288).mean(), 'plan_s', f'{time.time()-t:.1f}', flush=True)
    del pl, pos, d
