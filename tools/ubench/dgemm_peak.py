import torch, time, os
torch.backends.cuda.matmul.allow_tf32 = False
print(torch.cuda.get_device_name(), os.cpu_count())
for n in (4096, 8192):
    a = torch.randn(n, n, dtype=torch.float64, device="cuda"); b = torch.randn(n, n, dtype=torch.float64, device="cuda")
    for _ in range(3): c = a @ b
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    best = 1e9
    for _ in range(10):
        e0.record(); c = a @ b; e1.record(); torch.cuda.synchronize(); best = min(best, e0.elapsed_time(e1))
    print(f"cuBLAS DGEMM {n}^3: {2*n**3/best/1e9:.1f} TFLOP/s (best of 10, {best:.2f} ms)")
    # sustained
    t0 = time.time(); k = 0
    e0.record()
    while time.time() - t0 < 3:
        c = a @ b; k += 1
        if k % 10 == 0: torch.cuda.synchronize()
    e1.record(); torch.cuda.synchronize()
    print(f"  sustained ({k} iters): {2*n**3*k/e0.elapsed_time(e1)/1e9:.1f} TFLOP/s")
