import ctypes, torch, sys
sys.path.insert(0, '.')
import __graft_entry__
torch.cuda.init()
lp = ctypes.CDLL(__graft_entry__.build_l2_probe())
g, m = ctypes.c_float(), ctypes.c_float()
for mode in (0, 1):
    lp.l2_probe_read_gbs2(ctypes.c_int64(48 << 20), ctypes.c_int32(256), ctypes.c_int32(mode), ctypes.byref(g), ctypes.byref(m))
