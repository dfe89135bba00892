import sys, time, json, torch
sys.path.insert(0, '.')
import paper_conf_ppopp_huzslmlwtj24_b200 as fk
def t(fn):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); fn(); e1.record(); torch.cuda.synchronize()
    return round(e0.elapsed_time(e1), 3)
for prec in (32, 64):
    blocks = [10240] * 100 + [3082]
    kf = fk.KalmanFilter(blocks, dict(block_size=10240, p_defer=15, precision=prec))
    N = sum(blocks)
    gs = torch.randn(20, N, dtype=torch.float64, device="cuda")
    w = torch.zeros(N, dtype=torch.float64, device="cuda")
    abe = torch.full((1,), 0.1, dtype=torch.float64, device="cuda")
    r = {}
    r["pass_only_fresh"] = [t(lambda: kf.pass_only(gs[0])) for _ in range(3)]
    r["update"] = [t(lambda i=i: kf.update(gs[i], abe, 5.0, w)) for i in range(18)]
    r["pass_only_after"] = [t(lambda: kf.pass_only(gs[1])) for _ in range(3)]
    r["pass_only_g"] = [t(lambda i=i: kf.pass_only(gs[i])) for i in range(3)]
    print(prec, json.dumps(r), flush=True)
    kf.close(); del kf; torch.cuda.empty_cache()
