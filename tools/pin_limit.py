"""How much host memory can one process pin (cudaHostRegister) on this box?  Registers 8 GB
chunks until a registration fails; prints the running total."""
import ctypes
import sys

import numpy as np
import torch

cudart = ctypes.CDLL("libcudart.so.12") if len(sys.argv) < 2 else ctypes.CDLL(sys.argv[1])
torch.cuda.init()
bufs = []
tot = 0
for i in range(40):
    a = np.empty(8 << 30, np.uint8)
    a[::4096] = 1
    rc = cudart.cudaHostRegister(ctypes.c_void_p(a.ctypes.data), ctypes.c_size_t(a.nbytes), 3)
    if rc != 0:
        print(f"register #{i} failed rc={rc} after {tot >> 30} GB pinned", flush=True)
        break
    bufs.append(a)
    tot += a.nbytes
    print(f"pinned {tot >> 30} GB", flush=True)
