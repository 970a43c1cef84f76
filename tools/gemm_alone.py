"""Two bf16 cuBLAS GEMMs (8192^3 and the GPT FC1 stage GEMM), 5 launches each: the
workload whose DRAM traffic tools/gpu/*.sh reads with ncu (how much HBM the GEMM
beside a swap needs)."""
import torch
a = torch.randn(8192, 8192, dtype=torch.bfloat16, device="cuda")
b = torch.randn(8192, 8192, dtype=torch.bfloat16, device="cuda")
c = torch.empty(8192, 8192, dtype=torch.bfloat16, device="cuda")
for _ in range(5):
    torch.matmul(a, b, out=c)
a2 = torch.randn(4096, 5120, dtype=torch.bfloat16, device="cuda")
b2 = torch.randn(5120, 20480, dtype=torch.bfloat16, device="cuda")
c2 = torch.empty(4096, 20480, dtype=torch.bfloat16, device="cuda")
for _ in range(5):
    torch.matmul(a2, b2, out=c2)
torch.cuda.synchronize()
