import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, paper_conf_ipps_tanitni14_b200 as bo
n, p = int(sys.argv[1]), int(sys.argv[2])
v = int(sys.argv[3])
c = bo.generate_tri(n, p, 1, torch.int32, bo.ROW_WISE)
out = bo.triangulation(c, bo.ROW_WISE, v)
torch.cuda.synchronize()
print("ok", n, p, v, out[:4].tolist())
