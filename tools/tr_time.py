import sys, statistics, torch, json
sys.path.insert(0, "/root/repo")
import paper_conf_ipps_tanitni14_b200 as bo
def t(fn, reps=20):
    for _ in range(3): fn()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
    return statistics.median(ts)
for rows, cols in [(1 << 20, 1024), (1024, 1 << 20), (1 << 22, 32), (1 << 16, 4096)]:
    x = bo.generate_prefix(cols, rows, 1, torch.int32, bo.ROW_WISE)
    y = torch.empty((cols, rows), dtype=torch.int32, device="cuda")
    ms = t(lambda: bo.transpose(x, out=y))
    ok = torch.equal(y[:, :7], x[:7].T) and torch.equal(y[:, -3:], x[-3:].T)
    print(json.dumps(dict(rows=rows, cols=cols, ms=round(ms, 4), tbs=round(2 * rows * cols * 4 / ms / 1e9, 3), ok=bool(ok))))
