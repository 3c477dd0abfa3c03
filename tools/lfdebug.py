"""Debug aid: parity + per-round stats of one config under given options (not a test)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import graphgen as gg, oracle
import paper_conf_ppopp_nasrebp13_b200 as p
t = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).cuda()
for spec in sys.argv[1:]:
    k, sd, opts = spec.split(":", 2)
    g = gg.config(int(k), s=1, scale_down=int(sd))
    o_ids, o_tot = oracle.kruskal(g.n, g.src, g.dst, g.w)
    with p.MSTGraph(g.n, t(g.src), t(g.dst), t(g.w)) as h:
        for kv in filter(None, opts.split(",")):
            a, b = kv.split("=")
            h.set_option(int(a), int(b))
        h.set_profiling(True)
        ids, cnt, tot = h.run()
        st = h.stats()
    ok = cnt == len(o_ids) and tot == o_tot and np.array_equal(ids.cpu().numpy(), o_ids)
    print(spec, "OK" if ok else f"MISMATCH cnt {cnt} vs {len(o_ids)} tot {tot} vs {o_tot}",
          "switch", st["light_switch_round"], "t", st["light_t"], "dense", st["dense_round"])
    print("   n_r", st["n_r"]); print("   a_r", st["a_r"]); print("   comp", st["compacted"])
    print("   ms", [round(x, 3) for x in st["round_filter_ms"]])
