import sys, torch
sys.path.insert(0, '.')
import graphgen as gg, paper_conf_hpdc_jaiganeshb18_b200 as ecl
g = gg.make_config("C5", seed=1, device="cuda")
h = ecl.Handle(0)
out = torch.empty(g.n, dtype=torch.int32, device="cuda")
def t(opts, K=10):
    for k,v in opts.items(): h.set_option(k, v)
    for _ in range(3): h.run(g.nindex, g.nlist, out=out)
    torch.cuda.synchronize()
    ev=[(torch.cuda.Event(True),torch.cuda.Event(True)) for _ in range(K)]
    for a,b in ev:
        a.record(); h.run(g.nindex, g.nlist, out=out); b.record()
    torch.cuda.synchronize()
    r=sorted(a.elapsed_time(b) for a,b in ev)
    h.set_option("timing",1); h.run(g.nindex, g.nlist, out=out); ph=h.timing(); h.set_option("timing",0)
    print(opts, "median %.3f min %.3f phases %.3f" % (r[K//2], r[0], sum(ph.values())))
    for k in opts: h.set_option(k, {"prejump":2}.get(k,0))
t({})
t({"prejump":0})
t({"prejump":0, "timing":1})
