import ctypes as C, numpy as np, torch
torch.cuda.init()
cu = C.CDLL("libcuda.so.1")
rt = C.CDLL("libcudart.so.12")
a = np.zeros(1 << 22, np.uint8)
def bid(p):
    v = C.c_ulonglong(0)
    r = cu.cuPointerGetAttribute(C.byref(v), 7, C.c_ulonglong(p))  # CU_POINTER_ATTRIBUTE_BUFFER_ID = 7
    return r, v.value
print("unregistered", bid(a.ctypes.data))
print("register", rt.cudaHostRegister(C.c_void_p(a.ctypes.data), C.c_size_t(a.nbytes), 3))
print("registered", bid(a.ctypes.data))
rt.cudaHostUnregister(C.c_void_p(a.ctypes.data))
rt.cudaHostRegister(C.c_void_p(a.ctypes.data), C.c_size_t(a.nbytes), 3)
print("re-registered", bid(a.ctypes.data))
t = torch.empty(1 << 20, dtype=torch.uint8, pin_memory=True)
print("pinned torch", bid(t.data_ptr()))
d = torch.empty(1 << 20, dtype=torch.uint8, device="cuda")
print("device", bid(d.data_ptr()))
