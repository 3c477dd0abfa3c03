import numpy as np, torch, sys
sys.path.insert(0, '.')
import graphgen, paper_conf_ppopp_nasrebp13_b200 as p
g = graphgen.config(4)
t = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).cuda()
with p.MSTGraph(g.n, t(g.src), t(g.dst), t(g.w)) as h:
    h.run(); st = h.stats()
    print(st["n_r"], st["light_switch_round"], st["member_ends"])
