import sys, json, torch
sys.path.insert(0, '.')
import paper_conf_ppopp_huzslmlwtj24_b200 as fk
blocks = [10240] * 100 + [3082]
N = sum(blocks)
for prec in (64, 32):
    for d in (1, 3, 5, 8, 11, 15, 16):
        kf = fk.KalmanFilter(blocks, dict(block_size=10240, p_defer=d, precision=prec))
        gs = torch.randn(4, N, dtype=torch.float64, device="cuda")
        w = torch.zeros(N, dtype=torch.float64, device="cuda")
        abe = torch.full((1,), 0.1, dtype=torch.float64, device="cuda")
        for i in range(d + 1):
            kf.update(gs[i % 4], abe, 5.0, w)
        n = 2 * (d + 1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize(); e0.record()
        for i in range(n):
            kf.update(gs[i % 4], abe, 5.0, w)
        e1.record(); torch.cuda.synchronize()
        print(json.dumps({"precision": prec, "p_defer": d, "ms_per_update": e0.elapsed_time(e1) / n}), flush=True)
        kf.close(); del kf, gs; torch.cuda.empty_cache()
