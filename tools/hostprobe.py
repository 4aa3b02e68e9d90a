import time, torch, sys
sys.path.insert(0, '.')
import paper_conf_ipps_tanitni14_b200 as bo
for layout, v in ((0, 0), (1, 0)):
    c = bo.generate_tri(16, 65536, 3, torch.int32, layout)
    out = torch.empty(65536, dtype=torch.int32, device="cuda")
    for _ in range(10): bo.triangulation(c, layout, v, out=out)
    torch.cuda.synchronize()
    torch.cuda._sleep(int(0.2 * 2e9))
    t = time.perf_counter()
    for _ in range(200): bo.triangulation(c, layout, v, out=out)
    dt = (time.perf_counter() - t) / 200
    torch.cuda.synchronize()
    print(f"layout {layout}: host {dt*1e6:.2f} us/call")
