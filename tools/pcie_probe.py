"""H2D bandwidth of a 2.4 GB pinned buffer: torch pin_memory, and an mmap'd THP-advised region
registered with cudaHostRegister."""
import ctypes, mmap, os, sys, time
import torch
n = 2400 * 1000 * 1000
def rate(a, b):
    r = []
    for _ in range(3):
        torch.cuda.synchronize(); t = time.perf_counter(); b.copy_(a, non_blocking=True); torch.cuda.synchronize()
        r.append(n / (time.perf_counter() - t) / 1e9)
    return [round(x, 1) for x in r]
b = torch.empty(n, dtype=torch.uint8, device="cuda")
a = torch.empty(n, dtype=torch.uint8).pin_memory(); a.fill_(1)
print("torch pin_memory", rate(a, b), flush=True)
del a
# THP-advised anonymous mapping, touched, then registered (page-locked) with CUDA
libc = ctypes.CDLL("libc.so.6", use_errno=True)
m = mmap.mmap(-1, n + (2 << 20), flags=mmap.MAP_PRIVATE | mmap.MAP_ANONYMOUS)
addr = ctypes.addressof(ctypes.c_char.from_buffer(m))
base = (addr + (2 << 20) - 1) & ~((2 << 20) - 1)
print("madvise", libc.madvise(ctypes.c_void_p(base), ctypes.c_size_t(n), 14), flush=True)  # MADV_HUGEPAGE
h = torch.frombuffer(m, dtype=torch.uint8, count=n, offset=base - addr)
h.fill_(1)
cudart = ctypes.CDLL("libcudart.so.12") if os.path.exists("/usr/local/cuda/lib64/libcudart.so.12") else None
err = torch.cuda.cudart().cudaHostRegister(h.data_ptr(), n, 0)
print("cudaHostRegister", err, flush=True)
print("THP + register", rate(h, b), flush=True)
try:
    print(open("/sys/kernel/mm/transparent_hugepage/enabled").read().strip(), open("/proc/meminfo").read().split("AnonHugePages:")[1].split("\n")[0].strip())
except Exception as e:
    print(e)
