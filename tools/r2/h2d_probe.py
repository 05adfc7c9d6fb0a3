import ctypes, time, numpy as np, torch
torch.cuda.init()
rt = ctypes.CDLL("libcudart.so.12") if False else None
import glob
cands = glob.glob("/usr/local/cuda/lib64/libcudart.so*") + glob.glob("/opt/prime-rl/.venv/lib/python3.12/site-packages/nvidia/cuda_runtime/lib/libcudart.so*")
rt = ctypes.CDLL(cands[0])
n = 4 << 30
a = np.ones(n // 8, dtype=np.float64)
d = torch.empty(n // 8, dtype=torch.float64, device="cuda")
def cp():
    torch.cuda.synchronize(); t = time.perf_counter()
    rt.cudaMemcpy(ctypes.c_void_p(d.data_ptr()), ctypes.c_void_p(a.ctypes.data), ctypes.c_size_t(n), 1)
    torch.cuda.synchronize(); return time.perf_counter() - t
for _ in range(2): print("pageable", round(cp(), 3))
t = time.perf_counter(); r = rt.cudaHostRegister(ctypes.c_void_p(a.ctypes.data), ctypes.c_size_t(n), 0); treg = time.perf_counter() - t
print("register rc", r, round(treg, 3))
for _ in range(2): print("registered", round(cp(), 3))
t = time.perf_counter(); rt.cudaHostUnregister(ctypes.c_void_p(a.ctypes.data)); print("unregister", round(time.perf_counter() - t, 3))
