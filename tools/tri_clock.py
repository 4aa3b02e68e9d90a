"""Per-phase cycle profile of the tiled triangulation kernel (development tool).
Build with NVCC_APPEND_FLAGS=-DBO_TRI_CLOCK into a separate .so, run with
BULKOBL_LIB=<that .so>: prints the share of warp time in the preload, D = 0 and
each tile-diagonal."""
import sys, os, ctypes
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_ipps_tanitni14_b200 as bo
L = bo.lib()
f = L.bulk_debug_tri_clock
f.argtypes = [ctypes.c_void_p, ctypes.c_int]
buf = (ctypes.c_ulonglong * 72)()
for n, v, dt in [(64, 20, torch.float32), (64, 22, torch.float32), (48, 22, torch.float32), (48, 20, torch.float32)]:
    c = bo.generate_tri(n, 65536, 4, dt, 0)
    out = torch.empty(65536, dtype=dt, device="cuda")
    bo.triangulation(c, 0, v, out=out); torch.cuda.synchronize()
    f(buf, 1)
    bo.triangulation(c, 0, v, out=out); torch.cuda.synchronize()
    f(buf, 0)
    vals = list(buf)
    NT = (n + 3) // 4
    tot = sum(vals[:NT + 1])
    print(n, v, "total Mcyc", round(tot / 1e6, 1), " ".join(f"{'pre' if i == 0 else 'D' + str(i - 1)}:{vals[i] / tot * 100:.1f}" for i in range(NT + 1)))
