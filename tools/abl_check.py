import sys, os, time
sys.path.insert(0, '/root/repo')
import torch, numpy as np
import graphgen as gg, oracle
import paper_conf_hpdc_jaiganeshb18_b200 as ecl
h = ecl.Handle(0)
for name in ["C2", "C4"]:
    g = gg.make_config(name, seed=6, scale_down={"C2": 6, "C4": 8}[name], device="cuda")
    g = gg.shuffle_rows(g, seed=2)
    exp, _ = oracle.bfs(*g.numpy())
    for init in (3, 1, 2):
        for jump in (4, 1, 2, 3):
            for fini in (3, 1, 2):
                print(name, init, jump, fini, end=' ', flush=True)
                h.set_option("init", init).set_option("jump", jump).set_option("fini", fini)
                t = time.time()
                out = h.run(g.nindex, g.nlist)
                torch.cuda.synchronize()
                ok = np.array_equal(out.cpu().numpy(), exp)
                print(ok, round(time.time() - t, 3), flush=True)
