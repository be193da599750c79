import torch
n = 4096
a = torch.rand(n, n, dtype=torch.float32, device="cuda"); b = torch.rand(n, n, dtype=torch.float32, device="cuda")
torch.backends.cuda.matmul.allow_tf32 = False
for _ in range(3): c = a @ b
torch.cuda.synchronize()
