import os, sys, time, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_liaolysshfyctzlq23_b200 import binding as mb
M, N, K = [int(v) for v in sys.argv[1:4]]
mode = int(sys.argv[4])
A = torch.randn(M, K, device="cuda").bfloat16(); B = torch.randn(N, K, device="cuda").bfloat16()
C = torch.zeros(M, N, device="cuda")
mb.debug_options(gemm_mode=mode)
for i in range(3):
    t = time.time(); mb.debug_gemm_ex(6, M, N, K, A, K, 1, B, K, 1, C, N); torch.cuda.synchronize()
    print(M, N, K, "mode", mode, "%.1f us" % ((time.time() - t) * 1e6), "err", ((C - A.float() @ B.float().t()).abs().max() / (A.float() @ B.float().t()).abs().max()).item(), flush=True)
