import torch
A = torch.randn(8192, 8192, dtype=torch.float64, device="cuda"); B = torch.randn(8192, 8192, dtype=torch.float64, device="cuda")
for _ in range(2): C = A @ B
torch.cuda.synchronize()
