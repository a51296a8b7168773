"""Is a host->device cudaMemcpyAsync from torch pinned memory asynchronous?  Times the issue (host wall
clock) and the completion of 64-MiB H2D copies from (a) torch pin_memory tensors, (b) cudaHostAlloc
memory, (c) pageable memory, with cudaPointerGetAttributes' view of each."""
import ctypes
import time

import torch

rt = ctypes.CDLL("libcudart.so.12") if False else None
try:
    rt = ctypes.CDLL("libcudart.so")
except OSError:
    import glob
    rt = ctypes.CDLL(sorted(glob.glob("/usr/local/cuda/lib64/libcudart.so*"))[0])


class Attr(ctypes.Structure):
    _fields_ = [("type", ctypes.c_int), ("device", ctypes.c_int), ("devicePointer", ctypes.c_void_p),
                ("hostPointer", ctypes.c_void_p)]


def attr(p):
    a = Attr()
    r = rt.cudaPointerGetAttributes(ctypes.byref(a), ctypes.c_void_p(p))
    return r, a.type


N = 64 << 20
dev = torch.empty(8 * N, dtype=torch.uint8, device="cuda")
s = torch.cuda.Stream()
srcs = {}
t = torch.zeros(8 * N, dtype=torch.uint8, pin_memory=True)
srcs["torch_pinned"] = t.data_ptr()
p = ctypes.c_void_p()
rt.cudaHostAlloc(ctypes.byref(p), ctypes.c_size_t(8 * N), 0)
srcs["cudaHostAlloc"] = p.value
pg = bytearray(8 * N)
srcs["pageable"] = ctypes.addressof(ctypes.c_char.from_buffer(pg))
rt.cudaMemcpyAsync.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_void_p]
for name, src in srcs.items():
    for rep in range(2):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for k in range(8):
            rt.cudaMemcpyAsync(dev.data_ptr() + k * N, src + k * N, N, 1, s.cuda_stream)
        t1 = time.perf_counter()
        s.synchronize()
        t2 = time.perf_counter()
    print(name, "attr", attr(src), f"issue {1e3 * (t1 - t0):.2f} ms, done {1e3 * (t2 - t0):.2f} ms, "
          f"{8 * N / (t2 - t0) / 1e9:.1f} GB/s")
