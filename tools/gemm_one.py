"""One qos_op_gemm_ex launch per (M, N, K, epi, ksplit) spec, for ncu captures:
  ncu ... python tools/gemm_one.py 256:4096:4096:add_f32:1 256:4096:4096:add_f32:2"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_goelmkar26_b200 import qoserve as q  # noqa: E402

torch.cuda.set_device(0)
for spec in sys.argv[1:]:
    M, N, K, epi, ks = spec.split(":")
    M, N, K, ks = int(M), int(N), int(K), int(ks)
    A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    B = (torch.randn(N, K, device="cuda") / K ** 0.5).to(torch.bfloat16)
    Cn = N // 2 if epi == "silu_gate" else N
    C = torch.zeros(M, Cn, device="cuda", dtype=torch.float32 if "f32" in epi else torch.bfloat16)
    for _ in range(2):
        q.qos_op_gemm_ex(A.data_ptr(), B.data_ptr(), C.data_ptr(), M, N, K, epi, None, ks, None)
    torch.cuda.synchronize()
print("done")
