import sys, numpy as np, torch
sys.path.insert(0, '.')
import lfgen, oracle
from paper_conf_icpp_0002s22_b200 import dist
A = lfgen.fem27_bricks(20); G = 2
bounds = dist.plan_bounds(A.rowptr, G)
comm = dist.Comm.loopback(G); parts = []
for r in range(G):
    rp, col, val = dist.row_slice(A, int(bounds[r]), int(bounds[r + 1]))
    parts.append(dist.Partition(torch.from_numpy(rp).cuda(), torch.from_numpy(col).cuda(), torch.from_numpy(val).cuda(), bounds, r, n=2))
dist.factor(parts, comm); dist.linear_forest(parts, comm)
outs = [p.forest_export() for p in parts]; torch.cuda.synchronize()
f = np.concatenate([o["forest"].cpu().numpy() for o in outs])
o = oracle.run_pipeline(A); pi = o["pi"]; pw = o["pi_w"]
print("bounds", bounds, "cycles gpu", [int(x["n_cycles"].item()) for x in outs], "oracle", o["n_cycles"])
bad = np.nonzero((f != o["forest"]).any(1))[0]
print("bad vertices", bad[:20], len(bad))
# component of the first bad vertex in pi
seen=set(); comp=[]; st=[int(bad[0])]
while st:
    x=st.pop()
    if x in seen: continue
    seen.add(x); comp.append(x); st += [int(y) for y in pi[x] if y>=0]
comp=sorted(comp)
iscyc = all((pi[x]>=0).all() for x in comp)
print("component size", len(comp), "cycle", iscyc, "ranks", sorted(set(int(np.searchsorted(bounds, x, 'right')-1) for x in comp)))
edges=set()
for x in comp:
    for s in range(2):
        if pi[x,s]>=0: edges.add((min(x,int(pi[x,s])),max(x,int(pi[x,s])), float(pw[x,s])))
emin=min(edges, key=lambda e:(e[2],-e[0],-e[1]))
print("weakest (oracle rule)", emin)
for x in comp:
    print(x, "pi", pi[x].tolist(), "w", pw[x].tolist(), "gpu", f[x].tolist(), "orc", o["forest"][x].tolist())
