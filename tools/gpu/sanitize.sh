# compute-sanitizer on one small training step in eager mode and in graph mode
python -m paper_conf_ppopp_huzslmlwtj24_b200.build > /dev/null
cat > /tmp/san_step.py <<'PY'
import sys, numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_ppopp_huzslmlwtj24_b200 as fk
from fixtures import get_config, make_dataset, init_weights, force_groups
wl = get_config("c1_cu32"); m = wl.model
opt = type(wl.opt)(**{**wl.opt.__dict__, "block_size": 1024, "p_defer": 1})
ds = make_dataset("c1_cu32", 4); na = len(ds["types"])
cu = lambda x, dt=torch.float64: torch.as_tensor(np.ascontiguousarray(x)).to(dt).cuda()
for graph in (False, True):
    ctx = fk.Context(m, opt, types=ds["types"], local_batch=4, global_batch=4, graph=graph)
    ctx.set_params(cu(init_weights(m, 3, float(ds["energy"].mean() / na))))
    for s in range(2):
        met = ctx.train_step(cu(ds["coord"]), cu(ds["box"]), cu(ds["energy"]), cu(ds["force"]), cu(force_groups(na, s, 7), torch.int32))
    ea, e, f, v = ctx.forward(cu(ds["coord"]), cu(ds["box"]))
    torch.cuda.synchronize()
    print("graph", graph, "flags", met.cpu().numpy()[7])
    ctx.close()
PY
for tool in memcheck racecheck synccheck initcheck; do
  echo "== $tool"; timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python /tmp/san_step.py 2>&1 | tail -6
done
