import numpy as np, sys
sys.path.insert(0, '.')
import graphgen
g = graphgen.config(4)
n = g.n
ph = np.fromfile('gpurun_out/phi.bin', np.int32)
s, d, w = g.src, g.dst, g.w
t = int(sys.argv[1])
L = (w <= t) & (s != d)
cross = ph[s[L]] != ph[d[L]]
print("light edges", L.sum(), "crossing components at the switch:", cross.sum())
alive = ph >= 0
sz = np.bincount(ph[alive])
print("comps", len(sz), "largest", sz.max(), "sizes hist (log2)", np.bincount(np.log2(sz[sz>0]).astype(int)))
