"""How long do the NVML clock queries take on this box (idle and under a GPU load)?"""
import threading
import time

import pynvml
import torch

pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(0)


def q():
    t = time.perf_counter()
    pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
    t1 = time.perf_counter()
    pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
    t2 = time.perf_counter()
    pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
    t3 = time.perf_counter()
    return (t1 - t) * 1e3, (t2 - t1) * 1e3, (t3 - t2) * 1e3


print("idle", [tuple(round(v, 3) for v in q()) for _ in range(5)])
a = torch.randn(8192, 8192, device="cuda")
torch.cuda.synchronize()
res = []
stop = threading.Event()


def loop():
    while not stop.is_set():
        res.append(q())
        time.sleep(0.02)


lat0 = []
for _ in range(200):                       # control: no sampling thread
    t = time.perf_counter()
    b = a @ a
    torch.cuda.synchronize()
    lat0.append((time.perf_counter() - t) * 1e3)
print("control matmul+sync ms: median", sorted(lat0)[len(lat0) // 2], "max", max(lat0))
th = threading.Thread(target=loop)
th.start()
lat = []
for _ in range(200):                       # short kernels + syncs: host latency per sync under sampling
    t = time.perf_counter()
    b = a @ a
    torch.cuda.synchronize()
    lat.append((time.perf_counter() - t) * 1e3)
stop.set()
th.join()
print("loaded", [tuple(round(v, 3) for v in r) for r in res[:10]], "max", max(max(r) for r in res))
print("matmul+sync ms: median", sorted(lat)[len(lat) // 2], "max", max(lat))
