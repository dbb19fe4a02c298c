"""Does any TMA-using library kernel run on this box?  One bf16 GEMM through
torch (cuBLAS / cuBLASLt picks an sm_100 kernel); run under
  ncu --metrics gpu__time_duration.sum,smsp__inst_executed_op_tma... python tools/tma_box_check.py
to see the kernel's name, and print whether the result is right."""
import torch

a = torch.randn(4096, 4096, device="cuda", dtype=torch.bfloat16)
b = torch.randn(4096, 4096, device="cuda", dtype=torch.bfloat16)
c = a @ b
ref = (a[:64].float() @ b.float())
err = (c[:64].float() - ref).abs().max().item() / ref.abs().max().item()
torch.cuda.synchronize()
print("bf16 gemm ok", err < 1e-2, err)
