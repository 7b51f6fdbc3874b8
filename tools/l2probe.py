import torch, ctypes
from cuda.bindings import runtime as rt
for a in ("cudaDevAttrMaxPersistingL2CacheSize","cudaDevAttrMaxAccessPolicyWindowSize","cudaDevAttrL2CacheSize"):
    print(a, rt.cudaDeviceGetAttribute(getattr(rt.cudaDeviceAttr, a), 0))
