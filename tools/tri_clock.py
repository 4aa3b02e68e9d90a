"""Per-phase cycle profile of the tiled triangulation kernel (development tool).
Build with NVCC_APPEND_FLAGS=-DBO_TRI_CLOCK into a separate .so and run with
BULKOBL_LIB=<that .so>: prints the cycles per warp-job of the preload, D = 0
and, per tile-diagonal, the dense part, the shuffle reduction, the fix-up and
the warp sync (the instrumentation itself adds ~40 %: read the shares)."""
import sys, os, ctypes
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_ipps_tanitni14_b200 as bo
L = bo.lib()
f = L.bulk_debug_tri_clock
f.argtypes = [ctypes.c_void_p, ctypes.c_int]
buf = (ctypes.c_ulonglong * 160)()
n, v = 64, 20
lay = int(sys.argv[1]) if len(sys.argv) > 1 else 0
c = bo.generate_tri(n, 65536, 4, torch.float32, lay)
out = torch.empty(65536, dtype=torch.float32, device="cuda")
bo.triangulation(c, lay, v, out=out); torch.cuda.synchronize()
f(buf, 1); bo.triangulation(c, lay, v, out=out); torch.cuda.synchronize(); f(buf, 0)
vals = list(buf)
tot = vals[0] + vals[1] + sum(vals[80:144]) + sum(vals[150:153])
print("total Mcyc", tot / 1e6, "per warp-job cycles", tot / 32768)
print("pre %.1f%%  D0 %.1f%%" % (vals[0] / tot * 100, vals[1] / tot * 100))
print("coop: barrier-in %.1f%%  copy %.1f%%  barrier-out %.1f%%" % tuple(vals[150 + i] / tot * 100 for i in range(3)))
for D in range(1, 16):
    d = vals[80 + 4 * D:84 + 4 * D]
    print("D%2d dense %5.0f shfl %5.0f fix %5.0f sync %5.0f  (cycles per warp-job)" % (D, *(x / 32768 for x in d)))
print("sum dense %.1f%% shfl %.1f%% fix %.1f%% sync %.1f%%" % tuple(sum(vals[80 + 4 * D + k] for D in range(1, 16)) / tot * 100 for k in range(4)))
