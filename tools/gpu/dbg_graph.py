import sys, torch, numpy as np
sys.path.insert(0, '.')
import paper_conf_ppopp_huzslmlwtj24_b200 as fk
from fixtures import get_config, make_dataset, init_weights, force_groups
cu = lambda x, dt=torch.float64: torch.as_tensor(np.ascontiguousarray(x)).to(dt).cuda()
wl = get_config("t2_tiny"); m = wl.model
opt = type(wl.opt)(**{**wl.opt.__dict__, "p_defer": 2})
B = wl.batch; ds = make_dataset("t2_tiny", B); na = len(ds["types"])
w0 = init_weights(m, 3, float(ds["energy"].mean() / na))
outs = []
for trial in range(3):
  for graph in (True, False):
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=B, global_batch=B, graph=graph)
    ctx.set_params(cu(w0))
    mets = []
    for step in range(5):
        groups = force_groups(na, step, 17, opt.force_groups, opt.atoms_per_group)
        mets.append(ctx.train_step(cu(ds["coord"]), cu(ds["box"]), cu(ds["energy"]), cu(ds["force"]), cu(groups, torch.int32)).clone())
    outs.append((graph, ctx.get_params().cpu(), torch.stack(mets).cpu()))
    ctx.close()
ref = outs[0]
for g, w, mt in outs:
    d = (mt - ref[2]).abs()
    print(g, "w eq", torch.equal(w, ref[1]), "met maxdiff per col", d.max(0).values.tolist())
