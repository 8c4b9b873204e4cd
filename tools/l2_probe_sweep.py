import ctypes, torch, sys
sys.path.insert(0, '.')
import __graft_entry__
torch.cuda.init()
lp = ctypes.CDLL(__graft_entry__.build_l2_probe())
for mode in (0, 1):
    for mb in (24, 48, 96, 200):
        for rb in ((64, 128, 256, 512) if mode == 0 else (256,)):
            g, m = ctypes.c_float(), ctypes.c_float()
            rc = lp.l2_probe_read_gbs2(ctypes.c_int64(mb << 20), ctypes.c_int32(rb), ctypes.c_int32(mode), ctypes.byref(g), ctypes.byref(m))
            print("mode", mode, "MB", mb, "row", rb, "GB/s %.0f" % g.value, "ms %.3f" % m.value, rc, flush=True)
